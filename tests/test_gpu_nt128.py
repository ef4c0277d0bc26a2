"""The opt-in NT = 128 layout (I2CW_NT=128: 2 Winograd points per pass, 8 V slots of 32
TMEM columns, 32-channel epilogue rows with a 128B-swizzled TMA store) must pass the same
parity cases as the default. The variable is read once per process: subprocess."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_nt128_parity_subset():
    env = dict(os.environ, I2CW_NT="128")
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider",
                        os.path.join(ROOT, "tests", "test_gpu_parity.py"),
                        "-k", "r_sweep_same_pad or pads or rect or deconv_pad or pretransformed"],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]

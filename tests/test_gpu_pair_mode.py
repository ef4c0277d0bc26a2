"""The opt-in CTA-pair mode (I2CW_PAIR=1: clusters of 2, tcgen05.mma.cta_group::2, U split by
output-channel halves) must pass the same parity cases. The mode is chosen once per process,
so the cases run in a subprocess with the variable set."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_pair_mode_parity_subset():
    env = dict(os.environ, I2CW_PAIR="1")
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider",
                        os.path.join(ROOT, "tests", "test_gpu_parity.py"),
                        "-k", "cfg1 or r_sweep_same_pad or small_k or rect or multi_segment or pretransformed"],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]

"""GPU accuracy and coverage cases the round-1 suite missed (VERDICT r01 "What's weak" 1-3):

* r = 8, 9 (alpha = 12) conv AND deconv at C = K = 256 and 512, on U[-1, 1] and on the
  paper's U[1, 2] (Table 3), every output element
  against the fp64 oracle under |err| <= 1e-4 * sum|x||w| (BASELINE.json north_star);
* every residue Q mod m of every r = 2..9, conv and deconv;
* K-chunked accumulation: the K loop split into chunks whose partial sums the
  TMA reduce-add combines, forced small with the i2cw_debug_set_kchunk test hook;
* concurrent K slices on small grids (api.cu run_fused): parity, determinism, and the same
  result as the unsliced path within the bound;
* the mean relative error on U[1, 2] (the paper's Table 3 metric) held to the band measured
  on B200 (the tcgen05 fp32 accumulator truncates once per MMA), so a
  precision regression fails.
"""
import numpy as np
import pytest
import torch

import paper_conf_icpp_zhangzxyw24_b200 as i2cw
from tests.gpu_util import assert_parity, run_case

pytestmark = pytest.mark.gpu


def _mean_rel(y, yr):
    return float(np.mean(np.abs(y.detach().cpu().double().numpy() - yr) / np.abs(yr)))


# (kind, N, H, W, C=K, r): H, W give several tile blocks and ragged width tails
LARGE_C = [(kind, r, c, dist) for kind in ("conv", "deconv") for r in (8, 9) for c in (256, 512)
           for dist in ("sym", "pos")]


@pytest.mark.parametrize("kind,r,c,dist", LARGE_C, ids=lambda v: str(v))
def test_alpha12_large_channels_every_element(kind, r, c, dist):
    lo, hi = (-1.0, 1.0) if dist == "sym" else (1.0, 2.0)
    # W = 13: Q mod m != 0 for both F(5,8) and F(4,9); two images, 11 rows
    p = r // 2
    y, yr, b = run_case(kind, 2, 11, 13, c, c, r, r, p, p, lo=lo, hi=hi)
    err = assert_parity(y, yr, b)
    print(f"{kind} r={r} C=K={c} U[{lo},{hi}]: max err/B {err:.3e} mean rel {_mean_rel(y, yr):.3e}")
    if c == 512 and r == 9:
        # the default K-chunk cap splits this K loop (NKS = 64 * 9 = 576 k-steps)
        assert i2cw.debug_plan(kind, 2, 11, 13, c, c, r, r, p, p)["NKC"] > 1


def _residue_cases():
    cases = []
    for r in range(2, 10):
        m = i2cw.plan(r, 8)[0]
        p = r // 2
        for kind in ("conv", "deconv"):
            for res in range(m):
                # conv: Q = W + 2p - r + 1; deconv: Q = W + r - 1 - 2p
                base = (2 * p - r + 1) if kind == "conv" else (r - 1 - 2 * p)
                W = next(w for w in range(3 * m + 1, 5 * m + 2) if (w + base) % m == res and w + base >= 2 * m)
                cases.append((kind, r, W, res))
    return cases


@pytest.mark.parametrize("kind,r,W,res", _residue_cases(), ids=lambda v: str(v))
def test_every_width_residue(kind, r, W, res):
    p = r // 2
    y, yr, b = run_case(kind, 1, 6, W, 8, 12, r, r, p, p)
    assert y.shape[2] % i2cw.plan(r, 8)[0] == res
    assert_parity(y, yr, b)


@pytest.mark.parametrize("r", [3, 5, 7, 9])
@pytest.mark.parametrize("kind", ["conv", "deconv"])
def test_k_chunked_accumulation(kind, r):
    """K loop split into chunks of <= 2*r k-steps (NCC = 5 channel chunks -> 3 K-chunks, the
    last one shorter): same bound as one accumulation, and deterministic."""
    old = i2cw.debug_set_kchunk(2 * r)
    try:
        p = r // 2
        pl = i2cw.debug_plan(kind, 2, 9, 23, 40, 36, r, r, p, p)
        assert pl["NKC"] == 3 and pl["CPC"] == 2
        y, yr, b = run_case(kind, 2, 9, 23, 40, 36, r, r, p, p)
        assert_parity(y, yr, b)
        y2, _, _ = run_case(kind, 2, 9, 23, 40, 36, r, r, p, p)
        assert torch.equal(y, y2)
    finally:
        i2cw.debug_set_kchunk(old)


def test_k_chunks_reduce_truncation_error():
    """With all-positive inputs the truncating accumulator's error grows with the accumulation
    length; chunking the same K loop lowers the mean error."""
    args = ("conv", 2, 10, 24, 256, 64, 3, 3, 1, 1)
    oldsl = i2cw.debug_set_kslices(1)  # one accumulation (no concurrent K slices on this small grid)
    try:
        y1, yr, _ = run_case(*args, lo=1.0, hi=2.0)
        old = i2cw.debug_set_kchunk(24)  # 96 k-steps -> 4 chunks of 24
        try:
            y4, _, _ = run_case(*args, lo=1.0, hi=2.0)
        finally:
            i2cw.debug_set_kchunk(old)
    finally:
        i2cw.debug_set_kslices(oldsl)
    e1, e4 = _mean_rel(y1, yr), _mean_rel(y4, yr)
    print(f"mean rel: one accumulation {e1:.3e}, 4 K-chunks {e4:.3e}")
    assert e4 < 0.6 * e1


# 4 slices (alpha 12, 3 passes), 2 slices (CTA pairs, whole units; split tail), 3 slices (r = 7)
KSLICE_CASES = [("conv", 1, 12, 20, 96, 64, 8, 4), ("conv", 1, 7, 7, 512, 512, 3, 1),
                ("deconv", 1, 9, 11, 256, 64, 5, 2), ("conv", 1, 10, 10, 256, 128, 7, 3)]


@pytest.mark.parametrize("kind,N,H,W,C,K,r,p", KSLICE_CASES, ids=lambda v: str(v))
def test_k_slices_small_grid(kind, N, H, W, C, K, r, p):
    """A per-GPU shard of a few images fills few SMs: the planner splits the K loop into
    concurrent slices summed by a fixed-order combine. Every element within the
    bound, bitwise repeatable, and close to the one-accumulation result."""
    pl = i2cw.debug_plan(kind, N, H, W, C, K, r, r, p, p)
    assert pl["KSL"] > 1, pl
    y, yr, b = run_case(kind, N, H, W, C, K, r, r, p, p)
    assert_parity(y, yr, b)
    y2, _, _ = run_case(kind, N, H, W, C, K, r, r, p, p)
    assert torch.equal(y, y2)
    old = i2cw.debug_set_kslices(1)
    try:
        assert i2cw.debug_plan(kind, N, H, W, C, K, r, r, p, p)["KSL"] == 1
        y1, _, _ = run_case(kind, N, H, W, C, K, r, r, p, p)
    finally:
        i2cw.debug_set_kslices(old)
    assert_parity(y1, yr, b)
    d = float((y.double().cpu() - y1.double().cpu()).abs().max())
    assert d <= 2e-4 * float(b.max()), d


# Mean relative error on U[1,2] (the paper's Table 3 metric) at C = K = 64 measured on B200 with
# the round-to-nearest V split (profiles/r02_accuracy_table.md); the limits are ~1.5x the
# measured values so a regression fails. The paper's SIMT fp32 reaches 1.4e-7..1.1e-6 (Gamma8);
# the tcgen05 accumulator's per-MMA truncation sets our floor.
MEAN_BAND = {2: 2.5e-6, 3: 2.7e-6, 4: 3.5e-6, 5: 4.5e-6, 6: 5e-6, 7: 6e-6, 8: 9e-6, 9: 1e-5}


@pytest.mark.parametrize("r", sorted(MEAN_BAND))
def test_mean_error_band_u12(r):
    y, yr, b = run_case("conv", 2, 16, 32, 64, 64, r, r, r // 2, r // 2, lo=1.0, hi=2.0)
    assert_parity(y, yr, b)
    e = _mean_rel(y, yr)
    print(f"r={r}: mean rel err {e:.3e} (limit {MEAN_BAND[r]:.1e})")
    assert e < MEAN_BAND[r]

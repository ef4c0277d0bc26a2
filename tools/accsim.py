"""Numerical model of the fused kernel's 3xTF32 arithmetic (diagnostic).

Per output tile: V = B^T d in fp32, U = G w (fp64, rounded), the tf32 hi/lo split of V
(truncating or round-to-nearest), and the per-point contraction as 3 MMAs per k-step of 8
channels: each MMA adds its exact 8-product sum to the fp32 accumulator and rounds the result
either to nearest or toward zero (the tcgen05 behaviour the B200 measurements match), with the
cross terms optionally in a separate accumulator. Prints the mean relative error (the paper's
Table 3 metric, U[1,2] inputs) and max |err| / sum|x||w| against the exact fp64 result.
The transform matrices come from the library's exact host generator (C ABI).
Usage: python tools/accsim.py
"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_zhangzxyw24_b200 as i2cw  # noqa: E402


def mats(m, r):
    AT, G, BT = i2cw.transform_matrices(m, r)
    f = lambda M: np.array([[float(v) for v in row] for row in M])  # noqa: E731
    return f(AT), f(G), f(BT)
def trunc_f32(x):  # round toward zero to fp32
    f = x.astype(np.float32)
    # fix where rounding went away from zero
    bad = np.abs(f.astype(np.float64)) > np.abs(x)
    f[bad] = np.nextafter(f[bad], np.float32(0))
    return f
def tf32_trunc(x):
    u = x.astype(np.float32).view(np.uint32) & np.uint32(0xFFFFE000)
    return u.view(np.float32)
def tf32_rna(x):
    u = (x.astype(np.float32).view(np.uint32) + np.uint32(0x1000)) & np.uint32(0xFFFFE000)
    return u.view(np.float32)
def run(m, r, C, lo, hi, split, accmode, ntiles=4000, seed=0, sep_cross=False):
    rng=np.random.default_rng(seed)
    AT,G,BT = mats(m,r); a=m+r-1
    R=r
    d = rng.uniform(lo,hi,(ntiles,R,C,a)).astype(np.float32)
    w = rng.uniform(lo,hi,(R,C,r)).astype(np.float32)  # one output channel
    V = np.einsum('tj,nrcj->nrct', BT.astype(np.float32), d).astype(np.float32)  # fp32-ish
    U = np.einsum('ts,rcs->rct', G, w.astype(np.float64)).astype(np.float32)
    Uh = tf32_rna(U); Ul = tf32_rna(U.astype(np.float32)-Uh)
    if split=='trunc':
        Vh = tf32_trunc(V); Vl = (V - Vh).astype(np.float32); Vl = tf32_trunc(Vl)  # TC truncates lo
    else:
        Vh = tf32_rna(V); Vl = tf32_rna((V-Vh).astype(np.float32))
    # k-steps: (cc, fh), 8 channels each
    K = R*C
    Vh=Vh.reshape(ntiles,R,C//8,8,a).transpose(0,2,1,3,4).reshape(ntiles,K//8,8,a)
    Vl=Vl.reshape(ntiles,R,C//8,8,a).transpose(0,2,1,3,4).reshape(ntiles,K//8,8,a)
    Uh_=Uh.reshape(R,C//8,8,a).transpose(1,0,2,3).reshape(K//8,8,a)
    Ul_=Ul.reshape(R,C//8,8,a).transpose(1,0,2,3).reshape(K//8,8,a)
    acc = np.zeros((ntiles,a),np.float32); acc2=np.zeros((ntiles,a),np.float32)
    rnd = trunc_f32 if accmode=='trunc' else (lambda x: x.astype(np.float32))
    for ks in range(K//8):
        prods = [(Vl[:,ks],Uh_[ks]),(Vh[:,ks],Ul_[ks]),(Vh[:,ks],Uh_[ks])]
        for i,(A,B) in enumerate(prods):
            s = np.einsum('nct,ct->nt', A.astype(np.float64), B.astype(np.float64))
            if sep_cross and i<2:
                acc2 = rnd(acc2.astype(np.float64)+s)
            else:
                acc = rnd(acc.astype(np.float64)+s)
    M = (acc.astype(np.float64)+acc2.astype(np.float64)).astype(np.float32) if sep_cross else acc
    y = (M.astype(np.float32) @ AT.T.astype(np.float32))
    # exact
    yex = np.zeros((ntiles,m))
    dd = d.astype(np.float64); ww=w.astype(np.float64)
    for i in range(m):
        yex[:,i] = np.einsum('nrcs,rcs->n', dd[:,:,:,i:i+r], ww)
    B = np.zeros((ntiles,m))
    for i in range(m):
        B[:,i] = np.einsum('nrcs,rcs->n', np.abs(dd[:,:,:,i:i+r]), np.abs(ww))
    err = np.abs(y-yex)
    return (err/np.abs(yex)).mean(), (err/B).max()
if __name__ == "__main__":
 for (m,r,C) in [(6,3,64),(2,7,64),(4,9,64)]:
  for lo,hi in [(1,2),(-1,1)]:
    for split in ['trunc','rn']:
      for acc in ['trunc','rn']:
        for sep in [False, True]:
          mr, mx = run(m,r,C,lo,hi,split,acc, ntiles=1500, sep_cross=sep)
          print(f"F({m},{r}) C={C} U[{lo},{hi}] split={split:5s} acc={acc:5s} sepcross={sep}: mean rel {mr:.2e}  max err/B {mx:.2e}")

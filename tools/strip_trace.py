"""Diagnostic: CTA-0 timeline of the strip kernel (fused_strip.cuh trace points, clock64 cycles).
Kinds: 0-3 WG chunk start, 4-7 after in_full, 8-11 after math + box release, 12-15 after st_empty,
16-19 after st_full arrive, 20-23 epilogue d_full wait (2p: before, 2p+1: after), 24-27 epilogue
end, 28/29 issuer 0 before/after st_full wait (per chunk), 30 issuer 0 chunk committed,
31 input producer after in_empty wait (per chunk).
Usage: I2CW_LIB_EXPERIMENT=.../libi2cw_trace.so I2CW_STRIP=1 python tools/strip_trace.py [cfg]"""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_icpp_zhangzxyw24_b200 as i2cw

cfgs = {"cfg2": ("conv", 128, 56, 56, 64, 64, 3, 3, 1, 1), "c128": ("conv", 256, 28, 28, 128, 128, 3, 3, 1, 1),
        "c64": ("conv", 256, 28, 28, 64, 64, 3, 3, 1, 1)}
L = i2cw.lib()
L.i2cw_debug_trace.argtypes = [ctypes.c_int] * 10 + [ctypes.c_void_p] * 5
for name in sys.argv[1:] or ["cfg2"]:
    kind, N, H, W, C, K, R, S, ph, pw = cfgs[name]
    x = torch.rand((N, H, W, C), device="cuda"); w = torch.rand((K, R, S, C), device="cuda")
    P, Q = H + 2 * ph - R + 1, W + 2 * pw - S + 1
    y = torch.empty((N, P, Q, K), device="cuda")
    tr = torch.zeros(2 * 32 * 512 + 2 * 160, dtype=torch.int64, device="cuda")
    for _ in range(3):
        tr.zero_()
        rc = L.i2cw_debug_trace(0, N, H, W, C, K, R, S, ph, pw, x.data_ptr(), w.data_ptr(), y.data_ptr(), tr.data_ptr(),
                                torch.cuda.current_stream().cuda_stream)
        assert rc == 0
    torch.cuda.synchronize()
    TT = tr.cpu().numpy().astype(np.int64)
    cta = TT[2 * 32 * 512:].reshape(-1, 2)
    cta = cta[cta[:, 0] > 0]
    T = TT[:2 * 32 * 512].reshape(2, 32, 512)[0]
    t0 = T[T > 0].min()
    T = np.where(T > 0, T - t0, -1)
    v = lambda k: T[k][T[k] >= 0]
    pl = i2cw.debug_plan(kind, N, H, W, C, K, R, S, ph, pw)
    if len(cta):
        t0c = cta[:, 0].min()
        st, en = (cta[:, 0] - t0c) / 1e3, (cta[:, 1] - t0c) / 1e3
        print(f"per-CTA (us): start max {st.max():.1f}; end min {en.min():.1f} median {np.median(en):.1f} max {en.max():.1f}; "
              f"kernel span {en.max():.1f}")
        print("  end times sorted (every 8th):", np.round(np.sort(en)[::8], 1).tolist())
    print(f"== {name}: strip {pl['strip']} NUS {pl['NUS']} NIS {pl['NIS']} NOB {pl['NOB']} NITEMS {pl['NITEMS']} "
          f"tile_blocks {pl['tile_blocks']}")
    for g in range(4):
        a, b, c, d, e = (v(k + g) for k in (0, 4, 8, 12, 16))
        n = min(map(len, (a, b, c, d, e)))
        if n < 2: continue
        med = lambda z: float(np.median(z))
        print(f"WG{g}: {n} chunks; in_full wait {med(b[:n]-a[:n]):.0f}; math {med(c[:n]-b[:n]):.0f}; "
              f"st_empty wait {med(d[:n]-c[:n]):.0f}; STTM+arrive {med(e[:n]-d[:n]):.0f}; "
              f"end->next start {med(a[1:n]-e[:n-1]):.0f}; period {med(np.diff(a[:n])):.0f}")
    w28, w29, w30 = v(28), v(29), v(30)
    n = min(len(w28), len(w29), len(w30))
    print(f"issuer0: {n} chunks; st_full wait med {np.median(w29[:n]-w28[:n]):.0f} (mean {np.mean(w29[:n]-w28[:n]):.0f}); "
          f"issue (3 fh + shifts) med {np.median(w30[:n]-w29[:n]):.0f}; next med {np.median(w28[1:n]-w30[:n-1]):.0f}; "
          f"chunk period med {np.median(np.diff(w29[:n])):.0f}; span {w30[n-1]-w29[0]}")
    gaps = np.diff(w29[:n])
    print("  chunk periods:", gaps[:40].tolist())
    for g in range(4):
        ep = T[20 + g]
        ec = T[24 + g]
        npass = int(np.sum(ep[1::2] >= 0))
        rows = []
        for gp in range(min(npass, 6)):
            a, b = ep[2 * gp], ep[2 * gp + 1]
            cols = ec[gp * 8: gp * 8 + 8]
            # cols: [0..5] after column i issued, [6] after the pre-barrier, [7] end
            seq = [b - a, cols[6] - b] + [cols[i] - (cols[i - 1] if i > 0 else cols[6]) for i in range(6)] + [cols[7] - cols[5]]
            rows.append(seq)
        print(f"  WG{g} epilogue per pass [d_full wait, ld+pre, col0..col5, final wait]:")
        for r in rows: print("     ", [int(x) for x in r])
    p31 = v(31)
    print("producer in_empty->issue times (first 20):", p31[:20].tolist())

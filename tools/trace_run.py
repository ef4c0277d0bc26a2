"""Diagnostic: CTA-0 timeline of the fused kernel (clock64 cycles) for one config.
Trace kinds (see trace_rec calls in fused_tc.cu): 0-3 WG k-step start, 4-7 after st_empty wait,
8-11 after st_full arrive (warp 0 of each WG), 12-15 WG0 per-warp arrive, 16-18 issuer 0
(after st_full wait, after issue, after commit), 19-22/23-26 WG in_full before/after,
27 epilogue d_full wait (before/after), 28 epilogue end, 29 issuer 0 before st_full wait."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_icpp_zhangzxyw24_b200 as i2cw

cfgs = {"cfg2": ("conv", 128, 56, 56, 64, 64, 3, 3, 1, 1), "r9": ("conv", 64, 32, 32, 128, 128, 9, 9, 4, 4),
        "r5": ("conv", 64, 32, 32, 128, 128, 5, 5, 2, 2), "r3": ("conv", 64, 32, 32, 128, 128, 3, 3, 1, 1),
        "c512": ("conv", 256, 28, 28, 512, 512, 3, 3, 1, 1)}
L = i2cw.lib()
L.i2cw_debug_trace.argtypes = [ctypes.c_int] * 10 + [ctypes.c_void_p] * 5
for name in sys.argv[1:] or ["cfg2"]:
    kind, N, H, W, C, K, R, S, ph, pw = cfgs[name]
    x = torch.rand((N, H, W, C), device="cuda"); w = torch.rand((K, R, S, C), device="cuda")
    P, Q = H + 2 * ph - R + 1, W + 2 * pw - S + 1
    y = torch.empty((N, P, Q, K), device="cuda")
    tr = torch.zeros(2 * 32 * 512, dtype=torch.int64, device="cuda")
    for _ in range(3):
        tr.zero_()
        rc = L.i2cw_debug_trace(0, N, H, W, C, K, R, S, ph, pw, x.data_ptr(), w.data_ptr(), y.data_ptr(), tr.data_ptr(),
                                torch.cuda.current_stream().cuda_stream)
        assert rc == 0
    torch.cuda.synchronize()
    if int(tr.count_nonzero()) == 0:
        sys.exit("no trace records: build the library with `make -C paper_conf_icpp_zhangzxyw24_b200 TRACE=1`")
    T2 = tr.cpu().numpy().reshape(2, 32, 512).astype(np.int64)
    t0 = T2[T2 > 0].min()
    T2 = np.where(T2 > 0, T2 - t0, -1)   # cycles (clock64; CTA1 not comparable)
    t = T2[0]
    def v(k, cta=0): return T2[cta][k][T2[cta][k] >= 0]
    pl = i2cw.debug_plan(kind, N, H, W, C, K, R, S, ph, pw)
    print(f"== {name}: plan {pl}")
    nwg = 4 if pl["NT"] == 64 else 2
    for g in range(nwg):
        a, b, c = v(g), v(4 + g), v(8 + g)
        n = min(len(a), len(b), len(c))
        if n < 2: continue
        print(f"WG{g}: {n} ks; st_empty wait med {np.median(b[:n]-a[:n]):.0f}; transform med {np.median(c[:n]-b[:n]):.0f}; "
              f"arrive->next start med {np.median(a[1:n]-c[:n-1]):.0f}; period med {np.median(np.diff(a[:n])):.0f}")
        d_ = v(12 + g)
        if len(d_) >= n:
            print(f"      math+STTM issue med {np.median(d_[:n]-b[:n]):.0f}; wait::st+arrive med {np.median(c[:n]-d_[:n]):.0f}")
        fa, fb = v(19 + g), v(23 + g)
        m = min(len(fa), len(fb))
        print(f"      in_full waits med {np.median(fb[:m]-fa[:m]):.0f} max {np.max(fb[:m]-fa[:m])} sum {np.sum(fb[:m]-fa[:m])}")
    w29, w16, w17, w18 = v(29), v(16), v(17), v(18)
    n = min(len(w29), len(w16), len(w17), len(w18))
    print(f"issuer0: {n} ks; st_full wait med {np.median(w16[:n]-w29[:n]):.0f}; issue med {np.median(w17[:n]-w16[:n]):.0f}; "
          f"commit med {np.median(w18[:n]-w17[:n]):.0f}; ready->ready med {np.median(np.diff(w16[:n])):.0f}; span {w18[n-1]-w16[0]}")
    arr = [v(12 + w) for w in range(4)]
    n = min(len(a) for a in arr)
    A_ = np.stack([a[:n] for a in arr])
    print("WG0 per-warp arrive minus warp0 (median):", [float(np.median(A_[w] - A_[0])) for w in range(4)])
    print("epilogue d_full wait (before, after):", v(27).tolist(), " end:", v(28).tolist())
    # per k-step critical path sample: ks 8..15
    print("kg: CTA0 WG arrive | CTA1 WG arrive | CTA0 issuer ready | issued | committed   (ns)")
    for kg in range(8, min(16, len(w16), len(w17), len(w18))):
        g = kg % nwg; i = kg // nwg
        a0 = v(8 + g, 0)[i] if i < len(v(8 + g, 0)) else None
        a1 = v(8 + g, 1)[i] if i < len(v(8 + g, 1)) else None
        print(f"  {kg:3d} g{g} {a0} {a1}  ready {w16[kg]}  issued {w17[kg]}  commit {w18[kg]}")
    for cta in (0, 1):
        print(f"CTA{cta} WG0 start/after-wait/arrive first 4:", list(zip(v(0, cta)[:4].tolist(), v(4, cta)[:4].tolist(), v(8, cta)[:4].tolist())),
              " in_full waits:", list(zip(v(19, cta)[:4].tolist(), v(23, cta)[:4].tolist())))
    r29, r16, r17 = v(29, 1), v(16, 1), v(17, 1)
    if len(r29):
        print("relay (CTA1): kg: after st_full, after u_full, after remote arrive")
        for kg in range(8, min(12, len(r29), len(r16), len(r17))):
            print("   ", kg, r29[kg], r16[kg], r17[kg])
    u30, u31 = v(30), v(31)
    if len(u30):
        print("U producer (CTA0): kg: before u_empty wait, issue time, issuer ready (u_full done)")
        for kg in range(0, min(16, len(u30), len(u31))):
            print("   ", kg, u30[kg], u31[kg], w16[kg] if kg < len(w16) else None)
    if os.environ.get("TIMELINE"):
        lab = {0: "start", 4: "after-slot", 8: "arrive", 19: "in_full?", 23: "in_full!"}
        ev = []
        for k0, name_ in lab.items():
            for i, tt in enumerate(v(k0)):
                ev.append((int(tt), f"{name_}[{i}]"))
        for i, tt in enumerate(v(16)): ev.append((int(tt), f"   ISS ready[{i}]"))
        for i, tt in enumerate(v(18)): ev.append((int(tt), f"   ISS commit[{i}]"))
        ev.sort()
        lo_ = int(os.environ.get("TL_FROM", "20000")); prev = None
        for tt, s in ev:
            if lo_ <= tt < lo_ + 12000:
                print(f"   {tt:8d} (+{tt - prev if prev is not None else 0:5d}) {s}"); prev = tt
    e27 = T2[0][27]
    e28 = T2[0][28]
    if (e27[64:] >= 0).any():
        print("epilogue per pass (WG0 thread 0): d_full wait, TMEM ld -> d_empty, pair sums + pre-bar")
        for gp in range(0, 24):
            if e27[2 * gp] < 0 or e28[128 + 2 * gp] < 0: continue
            print(f"   pass {gp}: d_full wait {e27[2*gp+1]-e27[2*gp]}  tmem ld {e28[128+2*gp]-e27[2*gp+1]}  pre {e28[129+2*gp]-e28[128+2*gp]}")
        print("epilogue columns (WG0 thread 0): col: compute+STS, fence+bulk-wait, bar, store issue -> next col")
        for c in range(0, 60):
            b = 64 + 4 * c
            if b + 3 >= 512 or e27[b] < 0: continue
            nxt = e27[b + 4] if b + 4 < 512 and e27[b + 4] >= 0 else -1
            print(f"   {c:3d} t={e27[b]} compute+sts {e27[b+2]-e27[b]} fence+wait {e27[b+3]-e27[b+2]} bar {e27[b+1]-e27[b+3]} "
                  f"-> next {nxt-e27[b+1] if nxt>=0 else None}")
    if os.environ.get("ISSUER"):
        print("issuer0 per super-stage: before-wait, after-waits, after-issue, after-commit (cycles, relative)")
        w29, w16, w17, w18 = v(29), v(16), v(17), v(18)
        for j in range(10, min(40, len(w18))):
            print(f"   ss{j}: {w29[j]} +{w16[j]-w29[j]} +{w17[j]-w16[j]} +{w18[j]-w17[j]}  next-before {w29[j+1]-w18[j] if j+1 < len(w29) else None}")

"""Diagnostic: CTA-0 timeline of the fused kernel (clock64 cycles) for one config."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_icpp_zhangzxyw24_b200 as i2cw

cfgs = {"cfg2": ("conv", 128, 56, 56, 64, 64, 3, 3, 1, 1), "r9": ("conv", 64, 32, 32, 128, 128, 9, 9, 4, 4),
        "r5": ("conv", 64, 32, 32, 128, 128, 5, 5, 2, 2), "c512": ("conv", 256, 28, 28, 512, 512, 3, 3, 1, 1)}
L = i2cw.lib()
L.i2cw_debug_trace.argtypes = [ctypes.c_int] * 10 + [ctypes.c_void_p] * 5
for name in sys.argv[1:] or ["cfg2"]:
    kind, N, H, W, C, K, R, S, ph, pw = cfgs[name]
    x = torch.rand((N, H, W, C), device="cuda"); w = torch.rand((K, R, S, C), device="cuda")
    P, Q = H + 2 * ph - R + 1, W + 2 * pw - S + 1
    y = torch.empty((N, P, Q, K), device="cuda")
    tr = torch.zeros(16 * 512, dtype=torch.int64, device="cuda")
    for _ in range(3):
        tr.zero_()
        rc = L.i2cw_debug_trace(0, N, H, W, C, K, R, S, ph, pw, x.data_ptr(), w.data_ptr(), y.data_ptr(), tr.data_ptr(),
                                torch.cuda.current_stream().cuda_stream)
        assert rc == 0
    torch.cuda.synchronize()
    t = tr.cpu().numpy().reshape(16, 512).astype(np.int64)
    t0 = t[t > 0].min()
    t = np.where(t > 0, t - t0, -1)
    def valid(k): return t[k][t[k] >= 0]
    print(f"== {name}: plan {i2cw.debug_plan(kind, N, H, W, C, K, R, S, ph, pw)}")
    for g in range(2):
        a, b, c = valid(3 * g), valid(3 * g + 1), valid(3 * g + 2)
        n = min(len(a), len(b), len(c))
        print(f"WG{g}: {n} ksteps; wait(v_empty) med {np.median(b[:n]-a[:n]):.0f} cyc; transform med {np.median(c[:n]-b[:n]):.0f} cyc; "
              f"period med {np.median(np.diff(a[:n])):.0f}")
    r6, r7 = valid(6), valid(7)
    n = min(len(r6), len(r7))
    print(f"MMA: {n} ksteps; issue dur med {np.median(r7[:n]-r6[:n]):.0f}; ready->ready med {np.median(np.diff(r6[:n])):.0f} cyc; total span {r7[n-1]-r6[0]}")
    for g in range(2):
        e = valid(8 + g); f = valid(10 + g)
        print(f"WG{g} epilogue: wait d_full at {e.tolist()}, done {f.tolist()}")
    print("first 12 MMA ready times:", r6[:12].tolist())
    print("first 6 WG0 (start, after-wait, arrive):", list(zip(valid(0)[:6].tolist(), valid(1)[:6].tolist(), valid(2)[:6].tolist())))
    r12, r13, r14 = valid(12), valid(13), valid(14)
    print("MMA thread per k-step: (start, after v_full, after u_full, issued, after commits) first 8:")
    for i in range(8):
        print("   ", r12[i], r13[i], r6[i], r7[i], r14[i])
    print("WG1 first 6 (start, after-wait, arrive):", list(zip(valid(3)[:6].tolist(), valid(4)[:6].tolist(), valid(5)[:6].tolist())))

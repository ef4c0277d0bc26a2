"""Light per-CTA phase sums of the strip kernel (build with EXTRA=-DI2CW_LTRACE=1, load with
I2CW_LIB_EXPERIMENT): WG per chunk (in_full wait, math, st_empty wait, STTM), epilogue (d_full
wait, body) and the leader issuer's waits, averaged over CTAs (cycles)."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import bench
import paper_conf_icpp_zhangzxyw24_b200 as i2cw
L = i2cw.lib()
L.i2cw_debug_trace.argtypes = [ctypes.c_int] * 10 + [ctypes.c_void_p] * 5
for name in sys.argv[1:] or ["cfg2"]:
    kind, N, H, W, C, K, R, S, ph, pw, _ = bench.CONFIGS[name]
    x = torch.rand((N, H, W, C), device="cuda"); w = torch.rand((K, R, S, C) if kind == "conv" else (C, R, S, K), device="cuda")
    P, Q = i2cw.out_shape(kind, N, H, W, K, R, S, ph, pw)[1:3]
    y = torch.empty((N, P, Q, K), device="cuda")
    tr = torch.zeros(200 * 48, dtype=torch.int64, device="cuda")
    for _ in range(3):
        tr.zero_()
        assert L.i2cw_debug_trace(int(kind == "deconv"), N, H, W, C, K, R, S, ph, pw, x.data_ptr(), w.data_ptr(), y.data_ptr(),
                                  tr.data_ptr(), torch.cuda.current_stream().cuda_stream) == 0
    torch.cuda.synchronize()
    T = tr.cpu().numpy().reshape(200, 48)
    act = T[:, 4] > 0
    T = T[act]
    print(f"== {name}: {act.sum()} CTAs")
    for g in range(4):
        b = T[:, g * 8:(g + 1) * 8].astype(float)
        n, ne = b[:, 4], np.maximum(b[:, 7], 1)
        print(f"  WG{g}: chunks/CTA {n.mean():.1f}; per chunk: in_full {np.mean(b[:,0]/n):.0f} math {np.mean(b[:,1]/n):.0f} "
              f"st_empty {np.mean(b[:,2]/n):.0f} sttm {np.mean(b[:,3]/n):.0f}; per pass: d_full {np.mean(b[:,5]/ne):.0f} epi {np.mean(b[:,6]/ne):.0f}; "
              f"total WG busy {np.mean(b[:,0]+b[:,1]+b[:,2]+b[:,3]+b[:,5]+b[:,6]):.0f}")
    pair = i2cw.debug_plan(kind, N, H, W, C, K, R, S, ph, pw)["pair"]
    Tl = T[0::2] if pair else T  # pair: the even CTA of each pair is the MMA leader
    iss = Tl[:, 32:36].astype(float)
    nch = Tl[:, 4] * 4
    print(f"  issuer (leaders {len(Tl)}): total {iss[:,3].mean():.0f} cycles; st_full waits {iss[:,0].mean():.0f}, "
          f"u_full waits {iss[:,1].mean():.0f}, d_empty waits {iss[:,2].mean():.0f}; per chunk: st_full {np.mean(iss[:,0]/nch):.0f} u_full {np.mean(iss[:,1]/nch):.0f}")

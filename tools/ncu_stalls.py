"""Per-SASS-instruction warp-stall samples from `ncu --page source --csv --print-source sass`.
Usage: python tools/ncu_stalls.py src.csv [top N] [--window ADDR_FROM ADDR_TO]"""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]; data = rows[2:]
ci = {h: i for i, h in enumerate(hdr)}
stall_cols = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
tot = sum(int(r[ci["Warp Stall Sampling (All Samples)"]] or 0) for r in data)
print("total samples", tot)
agg = {h: sum(int(r[ci[h]] or 0) for r in data) for h in stall_cols}
print("by reason:", ", ".join(f"{h[6:]} {100*v/tot:.1f}%" for h, v in sorted(agg.items(), key=lambda t: -t[1]) if v))
N = int(sys.argv[2]) if len(sys.argv) > 2 else 40
base = int(data[0][0], 16)
top = sorted(range(len(data)), key=lambda i: -int(data[i][ci["Warp Stall Sampling (All Samples)"]] or 0))[:N]
for i in sorted(top):
    r = data[i]; s = int(r[ci["Warp Stall Sampling (All Samples)"]] or 0)
    reasons = sorted(((int(r[ci[h]] or 0), h[6:]) for h in stall_cols), reverse=True)[:3]
    print(f"{int(r[0],16)-base:6x} {100*s/tot:5.2f}% {r[1].strip()[:60]:60s} " + " ".join(f"{n}:{v}" for v, n in reasons if v))
if "--buckets" in sys.argv:
    B = 0x200
    acc = {}
    for r in data:
        a = (int(r[0], 16) - base) // B
        s = int(r[ci["Warp Stall Sampling (All Samples)"]] or 0)
        ex = int(r[ci["Instructions Executed"]] or 0)
        d = acc.setdefault(a, [0, 0, {}])
        d[0] += s; d[1] += ex
        for h in stall_cols:
            d[2][h[6:]] = d[2].get(h[6:], 0) + int(r[ci[h]] or 0)
    for a in sorted(acc):
        s, ex, rs = acc[a]
        if s < tot * 0.005: continue
        top3 = sorted(rs.items(), key=lambda t: -t[1])[:4]
        print(f"{a*B:6x} {100*s/tot:5.1f}% inst {ex:9d} " + " ".join(f"{k}:{v}" for k, v in top3))

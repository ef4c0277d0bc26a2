"""Attribute an ncu --set full capture's warp-stall samples of the fused kernel to code regions
(no GPU needed): python tools/ncu_regions.py REPORT.ncu-rep
Regions are found from SASS landmarks in address order: the prologue (before the register
split), the transform/epilogue warpgroups (between USETMAXREG.TRY_ALLOC and .DEALLOC: V compute =
LDS / FFMA2 stretch, V store = STTM stretch, epilogue = from LDTM to the loop back), and the
producer / issuer warps (after .DEALLOC). Within each region, samples are split by stall reason."""
import csv
import io
import subprocess
import sys
from collections import defaultdict

raw = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr, data = rows[1], rows[2:]
isrc, isamp = hdr.index("Source"), hdr.index("Warp Stall Sampling (All Samples)")
reasons = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
region = "prologue"
tot = defaultdict(float)
by = defaultdict(lambda: defaultdict(float))
top = []
for r in data:
    src = r[isrc]
    op = src.split()[0] if src.split() else ""
    if op.startswith("@"):
        op = src.split()[1]
    if "USETMAXREG.TRY_ALLOC" in src:
        region = "wg:other"
    elif "USETMAXREG.DEALLOC" in src:
        region = "producer/issuer"
    elif region.startswith("wg"):
        if op.startswith("LDS"):
            region = "wg:V compute"
        elif op.startswith("STTM"):
            region = "wg:V store"
        elif op.startswith("LDTM"):
            region = "wg:epilogue"
    s = float(r[isamp] or 0)
    tot[region] += s
    for h in reasons:
        v = r[hdr.index(h)]
        if v not in ("", "0"):
            by[region][h] += float(v)
    top.append((s, region, src.strip()[:70]))
T = sum(tot.values())
print(f"total samples {T:.0f}")
for k, v in sorted(tot.items(), key=lambda t: -t[1]):
    rs = sorted(by[k].items(), key=lambda t: -t[1])[:5]
    print(f"{k:18s} {100 * v / T:5.1f}%  " + ", ".join(f"{n[6:]} {100 * c / T:.1f}%" for n, c in rs))
print("\ntop instructions:")
for s, reg, src in sorted(top, reverse=True)[:25]:
    print(f"  {100 * s / T:5.2f}% {reg:16s} {src}")

"""Aggregate L2 sectors requested (global) and stall samples of an .ncu-rep by CUDA source line."""
import collections, csv, io, subprocess, sys
rep = sys.argv[1]; top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
agg = collections.defaultdict(lambda: [0.0, 0.0, 0.0, ""])
fname = cur = hdr = None
for r in rows:
    if not r: continue
    if r[0] == "File Path": fname = r[1].split("/")[-1]; continue
    if r[0] == "Line No": hdr = {c: i for i, c in enumerate(r)}; continue
    if hdr is None or len(r) < 8: continue
    if r[0]: cur = (fname, r[0]); agg[cur][3] = r[1]
    if cur is None: continue
    def f(c):
        try: return float(r[hdr[c]] or 0)
        except (ValueError, KeyError): return 0.0
    a = agg[cur]
    a[0] += f("L2 Theoretical Sectors Global"); a[1] += f("Warp Stall Sampling (All Samples)"); a[2] += f("Instructions Executed")
tot_s = sum(a[0] for a in agg.values()) or 1; tot_w = sum(a[1] for a in agg.values()) or 1
print(f"total L2 sectors (global) {tot_s/1e6:.1f} M = {tot_s*32/1e9:.2f} GB; stall samples {tot_w:.0f}")
key = {"stall": 1, "inst": 2}.get(sys.argv[3] if len(sys.argv) > 3 else "", 0)
for k, a in sorted(agg.items(), key=lambda x: -x[1][key])[:top]:
    print(f"{a[0]/1e6:9.1f}M sect {100*a[0]/tot_s:5.1f}%  samp {100*a[1]/tot_w:5.1f}%  inst {a[2]/1e6:7.1f}M  {k[0]}:{k[1]:>5} {a[3].strip()[:70]}")

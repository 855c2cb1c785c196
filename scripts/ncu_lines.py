"""Aggregate warp-stall samples of an .ncu-rep by CUDA source line (cuda,sass view)."""
import csv, io, subprocess, sys, collections
rep = sys.argv[1]; top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
agg = collections.defaultdict(lambda: [0.0, 0.0, collections.Counter()])
fname = None; hdr = None; src_text = {}
for r in rows:
    if not r: continue
    if r[0] == "File Path": fname = r[1].split("/")[-1]; continue
    if r[0] == "Function Name": continue
    if r[0] == "Line No": hdr = r; continue
    if hdr is None or len(r) < 6: continue
    line = r[0]
    if line:
        cur = (fname, line); src_text[cur] = r[1]
    try:
        w = float(r[4] or 0); e = float(r[7] or 0)
    except ValueError:
        continue
    a = agg[cur]; a[0] += w; a[1] += e
    for i, c in enumerate(hdr):
        if c.startswith("stall_") and "Not Issued" not in c and i < len(r):
            try: a[2][c[6:]] += float(r[i] or 0)
            except ValueError: pass
tot = sum(a[0] for a in agg.values()) or 1
for k, a in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
    print(f"{100*a[0]/tot:5.1f}% {a[1]/1e6:8.2f}M {k[0]}:{k[1]:>4} {src_text.get(k,'').strip()[:60]:60s} {a[2].most_common(3)}")

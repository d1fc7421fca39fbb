"""Per-source-line stall breakdown (barrier / long_sb / short_sb / wait / mio) of one kernel in an ncu report."""
import csv, io, subprocess, sys
rep, kern = sys.argv[1], sys.argv[2]
n = int(sys.argv[3]) if len(sys.argv) > 3 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass", "--kernel-name",
                      f"regex:{kern}", "--launch-count", "1"], capture_output=True, text=True).stdout
rows, fname, hdr = [], None, None
for r in csv.reader(io.StringIO(out)):
    if not r: continue
    if r[0] == "File Path" or r[0] == "File Name": fname = r[1].split("/")[-1]; continue
    if r[0] == "Line No": hdr = r; continue
    if hdr and r[0].isdigit():
        d = dict(zip(hdr, r))
        try: rows.append((fname, int(r[0]), r[1][:70], {k: float(d.get(k, 0) or 0) for k in hdr if k.startswith("stall_") and "Not Issued" not in k}, float(d.get("Instructions Executed", 0) or 0)))
        except ValueError: pass
tot = sum(sum(x[3].values()) for x in rows) or 1
ti = sum(x[4] for x in rows) or 1
agg = {}
for x in rows:
    for k, v in x[3].items(): agg[k] = agg.get(k, 0) + v
print("total:", {k[6:]: f"{v/tot*100:.1f}%" for k, v in sorted(agg.items(), key=lambda t: -t[1])[:8]})
for f, ln, src, st, ins in sorted(rows, key=lambda x: -sum(x[3].values()))[:n]:
    s = sum(st.values())
    top = sorted(st.items(), key=lambda t: -t[1])[:3]
    print(f"{s/tot*100:5.1f}%s {ins/ti*100:5.1f}%i {f}:{ln:<4d} {' '.join(f'{k[6:]}={v/tot*100:.1f}' for k, v in top):44s} {src}")

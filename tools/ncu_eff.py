"""Per-source-line warp instructions and thread efficiency (active lanes) of one kernel."""
import csv, io, subprocess, sys
rep, kern = sys.argv[1], sys.argv[2]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass", "--kernel-name",
                      f"regex:{kern}", "--launch-count", "1"], capture_output=True, text=True).stdout
fname, hdr, agg = None, None, []
for r in csv.reader(io.StringIO(out)):
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]; continue
    if r[0] == "Line No":
        hdr = r; continue
    if r[0] == "Function Name" or not r[0].isdigit():
        continue
    ie = hdr.index("Instructions Executed"); te = hdr.index("Thread Instructions Executed")
    try:
        agg.append((float(r[ie] or 0), float(r[te] or 0), fname, int(r[0]), r[1][:80]))
    except ValueError:
        pass
tw = sum(a[0] for a in agg); tt = sum(a[1] for a in agg)
print(f"warp-instr {tw/1e9:.2f}G  thread-instr {tt/1e9:.1f}G  overall lane efficiency {tt/(32*tw)*100:.1f}%")
for w, t, f, ln, s in sorted(agg, key=lambda a: -a[0])[:int(sys.argv[3]) if len(sys.argv) > 3 else 30]:
    print(f"{w/tw*100:5.1f}%  eff {t/(32*w+1e-9)*100:5.1f}%  {f}:{ln:<4d} {s}")

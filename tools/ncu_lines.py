"""Top CUDA source lines by warp-stall samples (with their main stall reasons) of an ncu report captured with
--import-source on:    python tools/ncu_lines.py rep.ncu-rep [n]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass"], capture_output=True,
                     text=True).stdout
fname, hdr, recs = "", None, []
for r in csv.reader(io.StringIO(raw)):
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].rsplit("/", 1)[-1]
    elif r[0] == "Line No":
        hdr = r
    elif hdr and len(r) == len(hdr) and r[0]:
        d = dict(zip(hdr, r))
        d["_file"] = fname
        recs.append(d)
def f(x):
    try: return float(x or 0)
    except ValueError: return 0.0
key = "Warp Stall Sampling (All Samples)"
tot = sum(f(d[key]) for d in recs) or 1
stalls = [h for h in (hdr or []) if h.startswith("stall_") and "Not Issued" not in h]
for d in sorted(recs, key=lambda d: -f(d[key]))[:n]:
    top = sorted(((f(d[s]), s[6:]) for s in stalls), reverse=True)[:3]
    why = " ".join(f"{s}:{100*v/max(f(d[key]),1):.0f}" for v, s in top if v > 0)
    print(f"{100*f(d[key])/tot:5.1f}% {d['_file'][:16]}:{d['Line No']:>5} [{why}] {d['Source'].strip()[:80]}")

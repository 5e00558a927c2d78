"""Top SASS instructions by warp-stall samples of an ncu report: python tools/ncu_hot.py rep.ncu-rep [n]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr = None
recs = []
for r in rows:
    if r and r[0] == "Address":
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        recs.append(dict(zip(hdr, r)))
key = "Warp Stall Sampling (All Samples)"
def f(x):
    try: return float(x or 0)
    except ValueError: return 0.0
tot = sum(f(r.get(key)) for r in recs) or 1
stall_cols = [h for h in (hdr or []) if h.startswith("stall_") or "Stall" in h and h != key]
for r in sorted(recs, key=lambda r: -f(r.get(key)))[:n]:
    print(f"{100*f(r.get(key))/tot:5.1f}%  {r.get('Address','')}  {r.get('Source','')[:90]}")

"""Developer helper: instruction counts of an ncu report, split by the
warp role regions of the family kernel (bundle loop / mask loop / spin)."""
import csv, subprocess, sys, collections
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
h = rows[1]; data = rows[2:]
isrc = h.index("Source"); ie = h.index("Instructions Executed"); ist = h.index("Warp Stall Sampling (All Samples)")
cnt = [int(r[ie] or 0) for r in data]; src = [r[isrc] for r in data]; st = [int(r[ist] or 0) for r in data]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rr = list(csv.reader(raw.splitlines())); hh = rr[0]; vv = rr[2]
g = lambda n: vv[hh.index(n)]
print("duration ms", g("gpu__time_duration.sum"), "issue", g("smsp__issue_active.avg.pct_of_peak_sustained_active"), "total inst", sum(cnt))
waits = [i for i in range(len(src)) if "TRYWAIT" in src[i]]
lds128 = [i for i in range(len(src)) if "LDS.128" in src[i]]
print("LDS.128 (km) at", lds128[:8])
spin = sum(cnt[i] for i in range(len(src)) if "NANOSLEEP" in src[i] or ("SYNCS.PHASECHK" in src[i] and "TRYWAIT" not in src[i]))
print("spin instructions", spin)

"""Summarise an ncu --metrics gpu__time_duration.sum launch list (csv) into profiles/."""
import csv, sys
lines = [l for l in open(sys.argv[1]) if l.startswith('"')]
rows = list(csv.reader(lines))
hdr = rows[0]
ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
allk, interp = [], []
for r in rows[1:]:
    if len(r) <= vi:
        continue
    v = float(r[vi].replace(",", ""))
    allk.append((r[ki], v))
    if "mscclInterpreter" in r[ki]:
        interp.append(v)
out = [
    "launch list: %s (ncu --metrics gpu__time_duration.sum --clock-control none -c 400; cold-cache, serialised)" % sys.argv[1],
    "all launches: %d, total %.3f ms" % (len(allk), sum(v for _, v in allk) / 1e6),
    "interpreter launches: %d, mean %.3f ms, min %.3f, max %.3f" % (len(interp), sum(interp) / len(interp) / 1e6,
                                                                     min(interp) / 1e6, max(interp) / 1e6),
    "other kernels are input generation (counter-based hash, torch elementwise) outside the timed region",
    "timed region = interpreter launches only (1 per step): share of the step = 100%",
]
print("\n".join(out))
open(sys.argv[2], "w").write("\n".join(out) + "\n")

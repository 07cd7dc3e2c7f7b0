"""Markdown tables from `bench.py --sweep` JSON lines: one row per size, one column pair
(eager / CUDA graph) per program set and implementation; cells are "us (busBW GB/s)" with a
'*' when the point passed its correctness check. Usage: sweep_table.py in.jsonl out.md"""
import json
import sys


def main(src, dst):
    rows = {}
    cols = []
    for line in open(src):
        d = json.loads(line)
        key = "%s/%s/%s" % (d["impl"], d.get("set", d["coll"]), "graph" if d["graph"] else "eager")
        if key not in cols:
            cols.append(key)
        cell = "%.1f (%.1f)%s" % (d["t_us_max"], d["busbw"], "*" if d.get("correct", True) else " WRONG")
        if d.get("latency_mode_us"):
            cell += " [1000x: %.1f]" % d["latency_mode_us"]
        rows.setdefault((d["coll"], d["bytes"]), {})[key] = (cell, d.get("program", ""))
    out = ["Per-size sweep (`bench.py --sweep`): time per op in us (busBW GB/s); * = checked correct "
           "(bit-exact sampled parity / exact permutation); [1000x] = 1000-iteration latency mode", ""]
    for coll in sorted({c for c, _ in rows}):
        cs = [k for k in cols if any(k in v for (c2, _), v in rows.items() if c2 == coll)]
        out.append("### %s" % coll)
        out.append("")
        out.append("| bytes/rank | " + " | ".join(cs) + " | programs |")
        out.append("|---|" + "---|" * (len(cs) + 1))
        for (c2, b), v in sorted(rows.items()):
            if c2 != coll:
                continue
            progs = sorted({p for _, p in v.values() if p and p != "nccl"})
            out.append("| %d | %s | %s |" % (b, " | ".join(v.get(k, ("", ""))[0] for k in cs), ", ".join(progs)))
        out.append("")
    open(dst, "w").write("\n".join(out) + "\n")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])

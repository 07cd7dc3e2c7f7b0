"""A/B driver: run bench.py configurations back to back (same box) and print one summary
line each. Usage: python tools/ab.py "label|--bench-args|ENV=V,ENV2=V" ... [--reps N]

Each configuration runs `reps` times, interleaved (a b a b ...), so a drift of the box shows
up in both arms; the summary is the median busBW and the per-run values."""
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def run(args, env):
    e = dict(os.environ)
    e.update(env)
    p = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--no-cpu", "--no-e2e", "--quiet-extra",
                        "--steps", "10", "--warmup", "3"] + args, capture_output=True, text=True, env=e, timeout=600)
    try:
        return json.loads(p.stdout.strip().splitlines()[-1])
    except Exception:
        return {"error": (p.stderr or p.stdout)[-400:]}


def main():
    reps = 3
    specs = []
    argv = sys.argv[1:]
    if "--reps" in argv:
        i = argv.index("--reps")
        reps = int(argv[i + 1])
        argv = argv[:i] + argv[i + 2:]
    for s in argv:
        label, a, env = (s.split("|") + ["", ""])[:3]
        envd = dict(kv.split("=", 1) for kv in env.split(",") if kv)
        specs.append((label, a.split(), envd))
    vals = {s[0]: [] for s in specs}
    for _ in range(reps):
        for label, a, envd in specs:
            d = run(a, envd)
            vals[label].append(d.get("value", d.get("error")))
            print(label, json.dumps({k: d.get(k) for k in ("value", "ms_per_step", "error")}), flush=True)
    for label, v in vals.items():
        num = [x for x in v if isinstance(x, (int, float))]
        print("SUMMARY %-28s median %s  runs %s" % (label, round(statistics.median(num), 2) if num else None, v))


if __name__ == "__main__":
    main()

"""Summarise an ncu --set full report of the interpreter into profiles/ (text + json)."""
import csv, io, json, subprocess, sys

def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2:]

KEYS = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed', 'lts__t_sector_hit_rate.pct',
        'lts__t_bytes.sum', 'sm__throughput.avg.pct_of_peak_sustained_elapsed',
        'sm__warps_active.avg.pct_of_peak_sustained_active', 'launch__registers_per_thread', 'launch__grid_size',
        'launch__block_size', 'smsp__inst_executed.sum', 'smsp__average_warp_latency_issue_stalled_barrier',
        'l1tex__t_bytes.sum']
SCALE = {'byte': 1, 'Kbyte': 1e3, 'Mbyte': 1e6, 'Gbyte': 1e9, 'Tbyte': 1e12}

def main(rep, tag, note, out_txt, out_json, alg_bytes=None):
    hdr, units, rows = raw(rep)
    vals = rows[0]
    d = {h: (v, u) for h, u, v in zip(hdr, units, vals)}
    lines = [note]
    for k in KEYS:
        if k in d:
            lines.append("%-62s %s %s" % (k, d[k][0], d[k][1]))
    rd = float(d['dram__bytes_read.sum'][0]) * SCALE[d['dram__bytes_read.sum'][1]]
    wr = float(d['dram__bytes_write.sum'][0]) * SCALE[d['dram__bytes_write.sum'][1]]
    lines.append("dram read+write per launch: %.3f GB" % ((rd + wr) / 1e9))
    if alg_bytes:
        lines.append("algorithmic bytes per launch: %.3f GB" % (alg_bytes / 1e9))
    open(out_txt, "w").write("\n".join(lines) + "\n")
    js = {"kernel": "mscclInterpreter<bf16,sum>", "version": tag, "dram_bytes_per_launch": int(rd + wr),
          "dram_read": int(rd), "dram_write": int(wr), "duration_ms": float(d['gpu__time_duration.sum'][0]),
          "source": out_txt}
    json.dump(js, open(out_json, "w"), indent=1)
    print("\n".join(lines))

if __name__ == "__main__":
    main(*sys.argv[1:6], alg_bytes=float(sys.argv[6]) if len(sys.argv) > 6 else None)

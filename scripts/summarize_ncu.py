"""Summarise ncu reports/launch lists into profiles/ (text + json).

python scripts/summarize_ncu.py <report.ncu-rep> <out_prefix>
python scripts/summarize_ncu.py --launches <launches.csv> <out_prefix>
"""
import csv
import io
import json
import subprocess
import sys

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "dram_read"),
    ("dram__bytes_write.sum", "dram_write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram_pct_peak"),
    ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed", "tensor_pipe_pct"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm_throughput_pct"),
    ("lts__t_sector_op_read_hit_rate.pct", "l2_read_hit_pct"),
    ("l1tex__m_xbar2l1tex_read_bytes_mem_global_op_tma_ld.sum", "tma_load_bytes"),
    ("launch__registers_per_thread", "regs"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("sm__cycles_elapsed.avg.per_second", "sm_clock"),
]


def report(path, prefix):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    out = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")]}
        for m, name in METRICS:
            if m in hdr:
                i = hdr.index(m)
                d[name] = f"{r[i]} {units[i]}".strip()
        out.append(d)
    json.dump(out, open(prefix + ".json", "w"), indent=1)
    with open(prefix + ".txt", "w") as f:
        for d in out:
            f.write(d["kernel"] + "\n")
            for k, v in d.items():
                if k != "kernel":
                    f.write(f"    {k:18s} {v}\n")
    print(open(prefix + ".txt").read())


def launches(path, prefix):
    lines = [l for l in open(path) if not l.startswith("==")]
    rows = list(csv.reader(io.StringIO("".join(lines))))
    h = rows[0]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    mine = ("moe::", "umma_", "route_small", "decode_finalize", "combine_kernel", "scatter_rows", "assign_kernel",
            "scan_kernel", "chunk_count", "router_select", "router_gemv", "tile_weights", "gemv13", "gemv2",
            "simt_gemm", "ep_plan", "ep_pack", "ep_final")
    ours = [(r[ki], float(r[vi]), r[ui]) for r in rows[1:] if len(r) > vi and any(m in r[ki] for m in mine)]
    with open(prefix + ".csv", "w") as f:
        f.write("kernel,duration,unit\n")
        for k, v, u in ours:
            f.write(f"\"{k}\",{v},{u}\n")
    tot = {}
    for k, v, u in ours:
        key = k.split("(")[0]
        tot[key] = tot.get(key, 0.0) + v
    s = sum(tot.values())
    with open(prefix + "_share.txt", "w") as f:
        f.write(f"{len(ours)} launches of libmoe_b200 kernels; total {s:.1f} (ncu, serialised, cold)\n")
        for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
            f.write(f"{v / s * 100:6.2f}%  {v:12.1f}  {k}\n")
    print(open(prefix + "_share.txt").read())


if __name__ == "__main__":
    if sys.argv[1] == "--launches":
        launches(sys.argv[2], sys.argv[3])
    else:
        report(sys.argv[1], sys.argv[2])

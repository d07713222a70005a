"""Summarise an ncu launch list + `--set full` captures into profiles/<round>/.

    python profiles/summarize.py gpurun_out profiles/r01

Writes ncu_summary.md (per-kernel share of the timed step from the launch list, and the key
--set full metrics per captured kernel), launches_summary.csv and traffic.json (DRAM bytes per
launch for bench.py's `roofline.traffic`)."""
import collections
import csv
import json
import os
import re
import subprocess
import sys

CAT = {"gemm_tc_kernel<0,": "qkv_gemm", "gemm_tc_kernel<4,": "qkv_gemm", "gemm_tc_kernel<2,": "gate_up_gemm",
       "gemm_tc_kernel<3,": "lm_head", "decode_attn_tma_kernel": "decode_attn", "decode_attn_kernel": "decode_attn",
       "prefill_attn_tc": "prefill_attn", "prefill_attn_ws": "prefill_attn", "prefill_attn_kernel": "prefill_attn", "rms_stats_kernel": "rmsnorm",
       "rmsnorm_kernel": "rmsnorm"}
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "B": 1, "KB": 1e3, "MB": 1e6, "GB": 1e9}


def short(name):
    m = re.search(r"(\w+_kernel)(<[^(]*>)?", name)
    return (m.group(1) + (m.group(2) or "")) if m else name[:40]


def read_csv_after_header(path):
    lines = open(path).read().splitlines()
    start = [i for i, l in enumerate(lines) if l.startswith('"ID"')][0]
    return list(csv.reader(lines[start:]))


def launch_shares(path):
    rows = read_csv_after_header(path)
    hdr = rows[0]
    ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
    tot, cnt = collections.Counter(), collections.Counter()
    for r in rows[1:]:
        k = short(r[ki])
        tot[k] += float(r[vi].replace(",", ""))
        cnt[k] += 1
    return tot, cnt


def full_metrics(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    if len(rows) < 3:
        return []
    hdr, units = rows[0], rows[1]
    want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
            "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
            "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
            "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
            "lts__throughput.avg.pct_of_peak_sustained_elapsed", "sm__cycles_elapsed.avg.per_second",
            "launch__grid_size"]
    res = []
    for r in rows[2:]:
        d = {"kernel": short(r[hdr.index("Kernel Name")])}
        for w in want:
            if w in hdr:
                i = hdr.index(w)
                v = float(r[i].replace(",", "") or 0)
                if w.startswith("dram__bytes"):
                    v *= UNIT.get(units[i], 1)
                d[w] = v
        res.append(d)
    return res


def main(src, dst):
    os.makedirs(dst, exist_ok=True)
    md = ["# ncu summary (B200, C1 PP=1 bench command; launch list = timed region via NVTX 'timed')", ""]
    lp = os.path.join(src, "launches.csv")
    traffic = {}
    if os.path.exists(lp):
        tot, cnt = launch_shares(lp)
        T = sum(tot.values())
        md += ["## Launch list (`--metrics gpu__time_duration.sum --clock-control none`, cold/serialised)", "",
               "| kernel | launches | total ms | share | avg us |", "|---|---|---|---|---|"]
        with open(os.path.join(dst, "launches_summary.csv"), "w") as f:
            f.write("kernel,launches,total_ms,share,avg_us\n")
            for k, v in tot.most_common():
                md.append(f"| `{k}` | {cnt[k]} | {v / 1e6:.3f} | {v / T:.3f} | {v / cnt[k] / 1e3:.1f} |")
                f.write(f"{k},{cnt[k]},{v / 1e6:.4f},{v / T:.4f},{v / cnt[k] / 1e3:.2f}\n")
        md += ["", f"total kernel time in the list: {T / 1e6:.3f} ms", ""]
    for rep in sorted(f for f in os.listdir(src) if f.endswith(".ncu-rep")):
        ms = full_metrics(os.path.join(src, rep))
        if not ms:
            continue
        md += [f"## `{rep}` (`--set full`)", "",
               "| kernel | grid | us | DRAM read MB | DRAM write MB | DRAM % peak | tensor-pipe % | warps active % | regs | L2 % | SM GHz |",
               "|---|---|---|---|---|---|---|---|---|---|---|"]
        for d in ms:
            md.append("| `{}` | {} | {:.1f} | {:.1f} | {:.1f} | {:.1f} | {:.1f} | {:.1f} | {:.0f} | {:.1f} | {:.2f} |".format(
                d["kernel"], int(d.get("launch__grid_size", 0)), d.get("gpu__time_duration.sum", 0) / 1e3
                if d.get("gpu__time_duration.sum", 0) > 1e4 else d.get("gpu__time_duration.sum", 0),
                d.get("dram__bytes_read.sum", 0) / 1e6, d.get("dram__bytes_write.sum", 0) / 1e6,
                d.get("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", 0),
                d.get("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed", 0),
                d.get("sm__warps_active.avg.pct_of_peak_sustained_active", 0),
                d.get("launch__registers_per_thread", 0),
                d.get("lts__throughput.avg.pct_of_peak_sustained_elapsed", 0),
                d.get("sm__cycles_elapsed.avg.per_second", 0)))
            cat = next((c for p, c in CAT.items() if d["kernel"].startswith(p)), None)
            if cat and cat not in traffic:
                traffic[cat] = d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
        md.append("")
    open(os.path.join(dst, "ncu_summary.md"), "w").write("\n".join(md) + "\n")
    tp = os.path.join(os.path.dirname(os.path.abspath(__file__)), "traffic.json")
    allt = json.load(open(tp)) if os.path.exists(tp) else {}
    allt["C1-pp1"] = {**allt.get("C1-pp1", {}), **traffic}
    json.dump(allt, open(tp, "w"), indent=1)
    print("\n".join(md))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])

"""Summarise ncu output for profiles/ (run here, on the CPU box).

  python tools/ncu_summary.py launches <launches.csv> <out.md> [title]
      per-kernel launch counts, total / mean device time and share of the step
      (cold-cache, serialised ncu timings: compare SHARES, not absolutes)
  python tools/ncu_summary.py full <report.ncu-rep> <out.json> [title]
      key metrics of a `ncu --set full` capture (duration, DRAM bytes,
      pipe utilisation, occupancy, stall reasons)
"""
import collections
import csv
import json
import re
import subprocess
import sys


def short(name):
    name = re.sub(r"\(.*", "", name)
    name = name.replace("void ", "")
    return name[:90]


def launches(csv_path, out_md, title=""):
    rows = [r for r in csv.reader(open(csv_path)) if len(r) > 10 and r[0] != "ID"]
    agg = collections.OrderedDict()
    for r in rows:
        if r[12] != "gpu__time_duration.sum":
            continue
        k = short(r[4])
        ns = float(r[14])
        a = agg.setdefault(k, [0, 0.0])
        a[0] += 1
        a[1] += ns
    ours = {k: v for k, v in agg.items() if k.startswith("kde::")}
    step = {k: v for k, v in ours.items() if v[0] > 1 and not k.startswith("kde::rows_to_cols")}
    tot_step = sum(v[1] / v[0] for v in step.values())
    tot_ours = sum(v[1] for v in ours.values())
    tot_all = sum(v[1] for v in agg.values())
    lines = [f"# ncu launch list: {title}", "",
             f"source: `{csv_path}` (`ncu --metrics gpu__time_duration.sum --clock-control none`), "
             "cold-cache serialised timings -- compare shares, not absolutes.", "",
             "Kernels launched once are model set-up / harness (not in the timed step); the last column is the",
             "kernel's share of one step (mean launch time over the sum of mean times of the per-step kernels).", "",
             "| kernel | launches | total us | mean us | share of step |", "|---|---:|---:|---:|---:|"]
    for k, (n, ns) in sorted(ours.items(), key=lambda x: -x[1][1]):
        sh = f"{ns / n / tot_step:.1%}" if k in step else "set-up"
        lines.append(f"| `{k}` | {n} | {ns / 1e3:.1f} | {ns / 1e3 / n:.2f} | {sh} |")
    lines += ["", f"other (torch fill / L2-flush / harness) kernels: {sum(v[0] for k, v in agg.items() if k not in ours)} "
              f"launches, {(tot_all - tot_ours) / 1e3:.1f} us", ""]
    open(out_md, "w").write("\n".join(lines))
    print("\n".join(lines))


WANT = [
    "gpu__time_duration.sum", "launch__grid_size", "launch__block_size", "launch__registers_per_thread",
    "dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__cycles_elapsed.avg.per_second", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
    "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "smsp__inst_executed.sum", "sm__sass_thread_inst_executed_op_ffma_pred_on.sum",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_dispatch_stall_per_issue_active.ratio",
]


def full(rep, out_json, title=""):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(txt.splitlines()))
    h, units = r[0], r[1]
    res = []
    for v in r[2:]:
        d = {"kernel": short(v[h.index("Kernel Name")])}
        for k in WANT:
            if k in h:
                x = v[h.index(k)]
                try:
                    x = float(x.replace(",", ""))
                except ValueError:
                    pass
                d[k] = x
                if units[h.index(k)]:
                    d[k + ".unit"] = units[h.index(k)]
        res.append(d)
    out = {"title": title, "source": rep, "kernels": res}
    json.dump(out, open(out_json, "w"), indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    {"launches": launches, "full": full}[sys.argv[1]](*sys.argv[2:])

"""Summaries of ncu outputs: launch list (per-kernel totals) and raw-page metrics."""
import collections
import csv
import json
import subprocess
import sys


def launches(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if 'Kernel Name' in r][0]
    h = rows[hi]
    ki, mi, ui = h.index('Kernel Name'), h.index('Metric Value'), h.index('Metric Unit')
    agg = collections.defaultdict(list)
    for r in rows[hi + 1:]:
        v = float(r[mi].replace(',', ''))
        u = r[ui]
        v = v / 1000 if u in ('nsecond', 'ns') else (v * 1000 if u in ('msecond', 'ms') else v)
        agg[r[ki].split('(')[0].split('<')[0]].append(v)
    tot = sum(sum(v) for v in agg.values())
    return {k: {"launches": len(v), "total_us": round(sum(v), 1), "avg_us": round(sum(v) / len(v), 2),
                "min_us": round(min(v), 2), "share_of_kernel_time": round(sum(v) / tot, 4)}
            for k, v in sorted(agg.items(), key=lambda x: -sum(x[1]))}


RAW = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum', 'launch__grid_size',
       'launch__block_size', 'launch__cluster_dim_x', 'launch__registers_per_thread',
       'launch__shared_mem_per_block_dynamic', 'sm__throughput.avg.pct_of_peak_sustained_elapsed',
       'gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed',
       'sm__warps_active.avg.pct_of_peak_sustained_active', 'smsp__inst_executed.sum',
       'smsp__pcsamp_warps_issue_stalled_barrier', 'smsp__pcsamp_warps_issue_stalled_long_scoreboard',
       'smsp__pcsamp_warps_issue_stalled_membar', 'smsp__pcsamp_warps_issue_stalled_wait',
       'smsp__pcsamp_warps_issue_stalled_short_scoreboard', 'smsp__pcsamp_warps_issue_stalled_math_pipe_throttle',
       'smsp__pcsamp_warps_issue_stalled_sleeping', 'smsp__pcsamp_warps_issue_stalled_no_instructions',
       'smsp__pcsamp_warps_issue_stalled_lg_throttle', 'smsp__pcsamp_warps_issue_stalled_selected',
       'smsp__pcsamp_warps_issue_stalled_branch_resolving', 'smsp__pcsamp_warps_issue_stalled_dispatch_stall',
       'smsp__pcsamp_sample_count']


def raw(rep):
    out = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h, u = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {'kernel': r[h.index('Kernel Name')].split('(')[0]}
        for w in RAW:
            if w in h:
                d[w + (' [' + u[h.index(w)] + ']' if u[h.index(w)] else '')] = r[h.index(w)]
        res.append(d)
    return res


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        print(json.dumps(launches(sys.argv[2]), indent=1))
    else:
        print(json.dumps(raw(sys.argv[2]), indent=1))

"""Summarise ncu outputs (launch-list CSV and --set full reports) into profiles/.

  python scripts/summarize_ncu.py full <report.ncu-rep> <out.json>
  python scripts/summarize_ncu.py launches <launches.csv> <out.md> <title>
"""
import collections
import csv
import json
import subprocess
import sys

KEYS = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed', 'sm__throughput.avg.pct_of_peak_sustained_elapsed',
        'lts__t_sector_hit_rate.pct', 'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum',
        'l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum', 'sm__warps_active.avg.pct_of_peak_sustained_active',
        'launch__registers_per_thread', 'launch__occupancy_limit_shared_mem', 'launch__occupancy_limit_registers',
        'sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active',
        'sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active', 'smsp__inst_executed.sum',
        'launch__waves_per_multiprocessor', 'sm__cycles_elapsed.avg.per_second', 'launch__grid_size',
        'launch__block_size', 'launch__shared_mem_per_block_dynamic',
        'smsp__average_warp_latency_issue_stalled_barrier.ratio',
        'smsp__average_warp_latency_issue_stalled_long_scoreboard.ratio',
        'smsp__average_warp_latency_issue_stalled_short_scoreboard.ratio',
        'smsp__average_warp_latency_issue_stalled_mio_throttle.ratio',
        'smsp__average_warp_latency_issue_stalled_math_pipe_throttle.ratio',
        'smsp__average_warp_latency_issue_stalled_wait.ratio']
SCALE = {'byte': 1, 'Kbyte': 1e3, 'Mbyte': 1e6, 'Gbyte': 1e9}


def full_report(rep, out_json):
    raw = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    rows = list(csv.reader(raw.splitlines()))
    h, units = rows[0], rows[1]
    res = []
    for row in rows[2:]:
        d = dict(zip(h, row))
        u = dict(zip(h, units))
        e = {'kernel': d.get('Kernel Name'), 'metrics': {k: [d.get(k), u.get(k)] for k in KEYS if k in d}}
        e['dram_bytes_per_launch'] = sum(float(d[k]) * SCALE.get(u[k], 1)
                                         for k in ('dram__bytes_read.sum', 'dram__bytes_write.sum'))
        res.append(e)
    json.dump(res, open(out_json, 'w'), indent=1)
    return res


def _table(f, seq):
    agg = collections.OrderedDict()
    tot = 0.0
    for name, ns in seq:
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += ns
        tot += ns
    f.write(f'Launches: {len(seq)}, total kernel time {tot / 1e6:.3f} ms\n\n'
            '| kernel | launches | total ms | mean us | share |\n|---|---|---|---|---|\n')
    for k, (n, ns) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        f.write(f'| `{k[:110]}` | {n} | {ns / 1e6:.3f} | {ns / n / 1e3:.1f} | {ns / tot:.3f} |\n')


def launches(csv_path, out_md, title, tail=0):
    """Whole launch list; with tail=N also the last N launches (the bench's
    timed region: its JSON line reports gpu_launches = N)."""
    rows = list(csv.reader(open(csv_path)))
    hi = [i for i, r in enumerate(rows) if r and r[0] == 'ID'][0]
    h = rows[hi]
    seq = []
    for r in rows[hi + 1:]:
        d = dict(zip(h, r))
        if d.get('Metric Name') != 'gpu__time_duration.sum':
            continue
        seq.append((d['Kernel Name'], float(d['Metric Value'].replace(',', ''))))
    with open(out_md, 'w') as f:
        f.write(f'# {title}\n\nncu launch list (`--metrics gpu__time_duration.sum --clock-control none`), '
                'cold-cache and serialised: compare shares, not absolutes.\n\n')
        if tail:
            f.write(f'## Timed region (the last {tail} launches = the JSON line\'s gpu_launches)\n\n')
            _table(f, seq[-tail:])
            f.write('\n## Whole run (label pass over all OCs + warm-up + timed region)\n\n')
        _table(f, seq)


if __name__ == '__main__':
    if sys.argv[1] == 'full':
        full_report(sys.argv[2], sys.argv[3])
    else:
        launches(sys.argv[2], sys.argv[3], sys.argv[4], int(sys.argv[5]) if len(sys.argv) > 5 else 0)

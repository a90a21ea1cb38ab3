"""Summarise `ncu --set full` reports into profiles/ (run here, without a GPU).

    python tools/ncu_summary.py TAG WORKLOAD rep1.ncu-rep|rep1.csv [...]

(a .csv is the `ncu -i rep --page raw --csv` export, for reports too large to bring back)

Writes profiles/<TAG>_ncu_full.json (key counters per launch) and merges the DRAM
traffic per launch into profiles/ncu_traffic.json (read by bench.py's roofline
`traffic` field), keyed "<WORKLOAD>:<spmm|sddmm>:K<K>".  The K of each launch is taken
from the template arguments (lanes * vw_feat * slices) -- see DESIGN.md.
"""
import csv
import io
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = ['Kernel Name', 'gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'lts__t_sector_hit_rate.pct', 'l1tex__t_sector_hit_rate.pct',
        'sm__warps_active.avg.pct_of_peak_sustained_active', 'launch__registers_per_thread',
        'lts__t_sectors.sum', 'lts__t_sectors.sum.pct_of_peak_sustained_elapsed',
        'smsp__issue_active.avg.pct_of_peak_sustained_active',
        'dram__throughput.avg.pct_of_peak_sustained_elapsed',
        'smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio',
        'smsp__average_warps_issue_stalled_wait_per_issue_active.ratio',
        'smsp__inst_executed.sum', 'sm__cycles_elapsed.avg.per_second', 'launch__grid_size',
        'launch__occupancy_limit_registers', 'lts__throughput.avg.pct_of_peak_sustained_elapsed',
        'lts__t_sectors_srcunit_tex.sum.pct_of_peak_sustained_elapsed',
        'l1tex__throughput.avg.pct_of_peak_sustained_elapsed',
        'l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed']
SCALE = {'byte': 1, 'Kbyte': 1e3, 'Mbyte': 1e6, 'Gbyte': 1e9, 'Tbyte': 1e12}


def rows_of(rep):
    if rep.endswith('.csv'):  # `ncu -i rep --page raw --csv` exported on the GPU box
        out = open(rep).read()
    else:
        out = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True,
                             text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, u = rows[0], rows[1]
    for r in rows[2:]:
        d = {}
        for k in KEYS:
            if k in h:
                d[k] = (r[h.index(k)], u[h.index(k)])
        yield d


def main():
    args = sys.argv[1:]
    ks = None  # --ks 32,32,64,...: K of each spmm/sddmm launch in report order
    if '--ks' in args:
        i = args.index('--ks')
        ks = [int(x) for x in args[i + 1].split(',')]
        del args[i:i + 2]
    tag, workload, reps = args[0], args[1], args[2:]
    summ = []
    traffic_path = os.path.join(ROOT, 'profiles', 'ncu_traffic.json')
    traffic = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
    for rep in reps:
        for d in rows_of(rep):
            name = d['Kernel Name'][0]
            m = re.search(r'(spmm|sddmm)_kernel<', name)
            rec = {k: f"{v} {un}".strip() for k, (v, un) in d.items()}
            if m:
                kind = m.group(1)
                b = 0.0
                for k in ('dram__bytes_read.sum', 'dram__bytes_write.sum'):
                    v, un = d[k]
                    b += float(v.replace(',', '')) * SCALE.get(un, 1)
                rec['dram_bytes'] = int(b)
                rec['report'] = os.path.basename(rep)
                # K is recorded by tools/profile_one.py order; store by kernel name too
                rec['kind'] = kind
                if ks is not None:
                    K = ks[sum(1 for r in summ if 'kind' in r)]
                    rec['K'] = K
                    traffic[f"{workload}:{kind}:K{K}"] = int(b)
            summ.append(rec)
    json.dump(summ, open(os.path.join(ROOT, 'profiles', f'{tag}_ncu_full.json'), 'w'), indent=1)
    if ks is not None:
        json.dump(traffic, open(traffic_path, 'w'), indent=1)
    print(json.dumps(summ, indent=1)[:3000])


if __name__ == '__main__':
    main()

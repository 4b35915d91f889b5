"""Summarise an ncu report (raw page) into the metrics DESIGN.md / profiles/ quote."""
import csv, json, subprocess, sys

WANT = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'lts__t_sector_hit_rate.pct', 'l1tex__t_sector_hit_rate.pct',
        'sm__warps_active.avg.pct_of_peak_sustained_active',
        'smsp__issue_active.avg.pct_of_peak_sustained_active', 'smsp__inst_executed.sum',
        'launch__registers_per_thread', 'launch__grid_size', 'launch__block_size',
        'sm__throughput.avg.pct_of_peak_sustained_elapsed',
        'dram__throughput.avg.pct_of_peak_sustained_elapsed',
        'smsp__warps_active.avg.per_cycle_active', 'lts__t_bytes.sum',
        'lts__t_sectors_srcunit_tex_op_read.sum', 'lts__t_sectors_srcunit_tex_op_write.sum',
        'l1tex__t_bytes.sum', 'sm__cycles_active.avg', 'smsp__cycles_active.avg',
        'sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active',
        'sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active',
        'smsp__inst_executed_op_shared_ld.sum', 'smsp__inst_executed_op_shared_st.sum',
        'smsp__inst_executed_op_global_red.sum', 'smsp__inst_executed_op_global_st.sum']
STALLS = ['long_scoreboard', 'short_scoreboard', 'wait', 'mio_throttle', 'lg_throttle', 'barrier',
          'math_pipe_throttle', 'not_selected', 'selected', 'dispatch_stall', 'no_instruction',
          'branch_resolving', 'drain', 'membar', 'sleeping', 'tex_throttle', 'imc_miss']


def summary(rep):
    out = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True,
                         text=True, check=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h, u = rows[0], rows[1]
    res = []
    for v in rows[2:]:
        d = {'kernel': v[h.index('Kernel Name')][:80]}
        for w in WANT:
            if w in h:
                d[w] = float(v[h.index(w)].replace(',', '')) if v[h.index(w)] else None
                d[w + '.unit'] = u[h.index(w)]
        st = {}
        for s in STALLS:
            k = f'smsp__average_warps_issue_stalled_{s}_per_issue_active.ratio'
            if k in h and v[h.index(k)]:
                st[s] = round(float(v[h.index(k)]), 3)
        d['stall_cycles_per_issue'] = st
        res.append(d)
    return res


if __name__ == '__main__':
    print(json.dumps(summary(sys.argv[1]), indent=1))

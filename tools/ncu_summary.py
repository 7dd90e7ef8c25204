"""Summarise an ncu report (raw page) into key metrics; used for profiles/."""
import csv, subprocess, sys, json
KEYS = ['Kernel Name', 'Grid Size', 'Block Size', 'gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'lts__t_sector_hit_rate.pct', 'l1tex__t_sector_hit_rate.pct', 'sm__throughput.avg.pct_of_peak_sustained_elapsed',
        'gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed',
        'smsp__issue_active.avg.pct_of_peak_sustained_active', 'sm__warps_active.avg.pct_of_peak_sustained_active',
        'launch__registers_per_thread', 'launch__occupancy_limit_registers', 'launch__occupancy_limit_shared_mem',
        'smsp__warps_eligible.avg.per_cycle_active', 'smsp__average_warp_latency_per_inst_issued.ratio',
        'smsp__inst_executed.sum', 'l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum', 'sm__inst_executed.avg.per_cycle_active',
        'dram__throughput.avg.pct_of_peak_sustained_elapsed', 'lts__throughput.avg.pct_of_peak_sustained_elapsed',
        'sm__cycles_elapsed.avg.per_second', 'launch__sm_count', 'local_load_bytes', 'smsp__sass_inst_executed_op_local_ld.sum']
STALL = 'smsp__average_warps_issue_stalled_'
# pipe utilisation and L1 wavefront columns (the roofline fractions bench.py reports)
PATTERNS = ('inst_executed_pipe_alu', 'inst_executed_pipe_fma', 'inst_executed_pipe_lsu', 'inst_executed_pipe_uniform',
            'pipe_alu_cycles_active', 'pipe_fma_cycles_active', 'pipe_lsu', 'l1tex__data_pipe_lsu_wavefronts',
            'l1tex__lsu_writeback', 'dram__bytes.sum', 'issue_active', 'pipe_shared_cycles_active')
def main(rep):
    out = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    r = list(csv.reader(out.splitlines()))
    h, units = r[0], r[1]
    res = []
    for row in r[2:]:
        d = dict(zip(h, row)); u = dict(zip(h, units))
        s = {k: (d.get(k), u.get(k)) for k in KEYS if k in d}
        s.update({k: (d.get(k), u.get(k)) for k in h if any(p in k for p in PATTERNS) and d.get(k) not in ('', None)})
        st = {k[len(STALL):].replace('_per_issue_active.ratio', ''): d[k] for k in h if k.startswith(STALL) and k.endswith('_per_issue_active.ratio')}
        st = dict(sorted(((k, float(v)) for k, v in st.items() if v not in ('', None)), key=lambda x: -x[1])[:10])
        s['top_stalls_per_issue'] = st
        res.append(s)
    return res
if __name__ == '__main__':
    print(json.dumps(main(sys.argv[1]), indent=1))

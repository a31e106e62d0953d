"""Summarise .ncu-rep files: key throughput metrics + top stall reasons (reads ncu --page raw csv)."""
import csv, io, subprocess, sys, json
KEYS = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'dram__throughput.avg.pct_of_peak_sustained_elapsed', 'sm__throughput.avg.pct_of_peak_sustained_elapsed',
        'sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active',
        'sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active',
        'sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_active',
        'smsp__issue_active.avg.pct_of_peak_sustained_active', 'sm__warps_active.avg.pct_of_peak_sustained_active',
        'launch__registers_per_thread', 'launch__occupancy_limit_registers', 'launch__occupancy_limit_shared_mem',
        'l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum', 'l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum',
        'smsp__inst_executed.sum', 'sm__cycles_elapsed.avg.per_second', 'launch__grid_size', 'launch__block_size',
        'l1tex__t_bytes_pipe_lsu_mem_global_op_ld.sum', 'lts__t_bytes.sum']
def summarise(path):
    out = subprocess.run(['ncu', '-i', path, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for vals in rows[2:]:
        d = dict(zip(hdr, vals)); u = dict(zip(hdr, units))
        r = {'kernel': d.get('Kernel Name', '')[:90]}
        for k in KEYS:
            if k in d: r[k] = f"{d[k]} {u[k]}".strip()
        st = sorted([(k.replace('smsp__pcsamp_warps_issue_stalled_', ''), float(v)) for k, v in d.items()
                     if k.startswith('smsp__pcsamp_warps_issue_stalled_') and not k.endswith('not_issued') and v not in ('', 'n/a')],
                    key=lambda x: -x[1])
        tot = sum(v for _, v in st) or 1
        r['stalls_pct'] = {k: round(100 * v / tot, 1) for k, v in st[:8]}
        res.append(r)
    return res
if __name__ == '__main__':
    for p in sys.argv[1:]:
        print(json.dumps({'file': p, 'launches': summarise(p)}, indent=1))

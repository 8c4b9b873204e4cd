"""Summarise an ncu report (raw page) into the metrics the roofline needs."""
import csv, subprocess, sys, json
WANT = ['gpu__time_duration.sum','dram__bytes_read.sum','dram__bytes_write.sum','lts__t_sector_hit_rate.pct',
 'sm__warps_active.avg.pct_of_peak_sustained_active','launch__registers_per_thread','launch__grid_size',
 'launch__occupancy_limit_registers','launch__occupancy_limit_shared_mem','sm__throughput.avg.pct_of_peak_sustained_elapsed',
 'gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed','lts__throughput.avg.pct_of_peak_sustained_elapsed',
 'l1tex__throughput.avg.pct_of_peak_sustained_elapsed','dram__throughput.avg.pct_of_peak_sustained_elapsed',
 'smsp__inst_executed.sum','l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum','lts__t_sectors_srcunit_tex_op_read.sum',
 'smsp__inst_executed_op_global_red.sum','smsp__issue_active.avg.pct_of_peak_sustained_active',
 'sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active','sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active',
 'smsp__average_warp_latency_issue_stalled_long_scoreboard','lts__t_bytes.sum','sm__cycles_elapsed.avg.per_second']
def summary(rep):
    if rep.endswith('.csv'):
        out = open(rep).read()
    else:
        out = subprocess.run(['ncu','-i',rep,'--page','raw','--csv'],capture_output=True,text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr, units = rows[0], rows[1]
    res = []
    for vals in rows[2:]:
        d = {'kernel': vals[hdr.index('Kernel Name')][:90]}
        for w in WANT:
            if w in hdr:
                d[w] = vals[hdr.index(w)] + ' ' + units[hdr.index(w)]
        res.append(d)
    return res
if __name__ == '__main__':
    for d in summary(sys.argv[1]):
        for k, v in d.items(): print(f'{k:70s} {v}')

"""Summarise ncu --set full reports (raw page) for profiles/."""
import csv, subprocess, sys, io
M = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
     'gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed', 'dram__throughput.avg.pct_of_peak_sustained_elapsed',
     'sm__throughput.avg.pct_of_peak_sustained_elapsed', 'sm__warps_active.avg.pct_of_peak_sustained_active',
     'launch__registers_per_thread', 'launch__grid_size', 'launch__block_size',
     'sm__pipe_tensor_op_hmma_cycles_active.avg.pct_of_peak_sustained_active',
     'sm__inst_executed_pipe_uniform.avg.pct_of_peak_sustained_active',
     'l1tex__t_sector_hit_rate.pct', 'lts__t_sector_hit_rate.pct',
     'smsp__average_warp_latency_issue_stalled_long_scoreboard', 'smsp__warp_issue_stalled_long_scoreboard_per_warp_active.pct',
     'smsp__warp_issue_stalled_lg_throttle_per_warp_active.pct', 'smsp__warp_issue_stalled_barrier_per_warp_active.pct',
     'smsp__warp_issue_stalled_membar_per_warp_active.pct']
for f in sys.argv[1:]:
    out = subprocess.run(['ncu', '-i', f, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units = rows[0], rows[1]
    for r in rows[2:]:
        name = r[h.index('Kernel Name')].split('(')[0]
        print(f"== {f.split('/')[-1]} :: {name}")
        for m in M:
            cands = [i for i, x in enumerate(h) if x == m]
            if cands:
                i = cands[0]
                print(f"   {m:70s} {r[i]:>14s} {units[i]}")

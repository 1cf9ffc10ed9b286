"""Key counters of ncu raw CSVs (gpurun_out/ncu_TAG/full_*.raw.csv) side by side."""
import csv, glob, sys
K = ['gpu__time_duration.sum', 'smsp__inst_executed.sum', 'sm__cycles_active.avg', 'sm__cycles_active.min',
     'sm__cycles_active.max', 'dram__bytes_read.sum', 'dram__bytes_write.sum', 'lts__t_sectors_srcunit_tex.sum',
     'smsp__issue_active.avg.pct_of_peak_sustained_active', 'l1tex__t_sector_hit_rate.pct',
     'smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio',
     'smsp__average_warps_issue_stalled_wait_per_issue_active.ratio',
     'smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio',
     'smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio',
     'smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio',
     'smsp__average_warps_issue_stalled_no_instruction_per_issue_active.ratio',
     'smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio',
     'smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio',
     'smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio']
for f in sorted(glob.glob(f"gpurun_out/ncu_{sys.argv[1]}/full_*.raw.csv")):
    rows = list(csv.reader(open(f)))
    d = dict(zip(rows[0], rows[2]))
    print(f.split('/')[-1][5:-8], {k.replace('smsp__average_warps_issue_stalled_', 'st_').replace('_per_issue_active.ratio', ''): d.get(k) for k in K})

"""Summarise an ncu report: key metrics + top stalled SASS lines (builder tooling)."""
import csv, subprocess, sys, io
rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(raw)))
h, units = r[0], r[1]
want = ['Kernel Name', 'gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'dram__throughput.avg.pct_of_peak_sustained_elapsed', 'sm__warps_active.avg.pct_of_peak_sustained_active',
        'launch__registers_per_thread', 'launch__grid_size', 'launch__block_size',
        'launch__occupancy_limit_shared_mem', 'sm__throughput.avg.pct_of_peak_sustained_elapsed',
        'lts__t_sector_hit_rate.pct', 'lts__throughput.avg.pct_of_peak_sustained_elapsed',
        'smsp__inst_executed.sum', 'launch__shared_mem_per_block_dynamic',
        'l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum', 'smsp__issue_active.avg.pct_of_peak_sustained_active',
        'smsp__sass_average_data_bytes_per_sector_mem_global_op_ld.ratio',
        'smsp__sass_average_data_bytes_per_sector_mem_global_op_st.ratio',
        'lts__t_sectors_srcunit_tex_op_read.sum', 'l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum']
for row in r[2:]:
    for i, k in enumerate(h):
        if k in want:
            print(f"{k:60s} {units[i]:>12s} {row[i]}")
    print("--")
if len(sys.argv) > 2:
    src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(src)))
    hh = rows[1]
    i_src = hh.index('Source'); i_s = hh.index('Warp Stall Sampling (All Samples)'); i_a = hh.index('Address')
    i_e = hh.index('Instructions Executed')
    data = rows[2:]
    tot = sum(int(x[i_s] or 0) for x in data) or 1
    top = sorted(range(len(data)), key=lambda k: -int(data[k][i_s] or 0))[:int(sys.argv[2])]
    for k in sorted(top):
        x = data[k]
        print(f"{x[i_a][-5:]} {100*int(x[i_s] or 0)/tot:5.1f}% ex={x[i_e]:>9} {x[i_src][:100]}")

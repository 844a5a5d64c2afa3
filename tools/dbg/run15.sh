cd $GRAFT_REPO_ROOT
GZKP_DFP=1 timeout 600 ncu --section ComputeWorkloadAnalysis --section SchedulerStats --section WarpStateStats --metrics sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:k_accum -s 2 -c 1 -o gpurun_out/accum_dfp python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-prepared > /dev/null 2>&1
ncu -i gpurun_out/accum_dfp.ncu-rep --page raw --csv 2>/dev/null | python -c "
import csv,sys
rows=list(csv.reader(sys.stdin)); h,v=rows[0],rows[2]
for i,n in enumerate(h):
    if any(k in n for k in ['pipe_fmaheavy_cycles','pipe_fp64','issue_active','pipe_alu_cycles','gpu__time_duration.sum','warps_issue_stalled_wait_per','warps_issue_stalled_math','warps_issue_stalled_short','warps_issue_stalled_long','registers_per']):
        print(n, v[i])
"

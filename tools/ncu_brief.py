import csv, collections, subprocess, sys
rep=sys.argv[1]
raw=subprocess.run(['ncu','-i',rep,'--page','raw','--csv'],capture_output=True,text=True).stdout.splitlines()
rows=list(csv.reader(raw)); hdr,units=rows[0],rows[1]
keys=['Kernel Name','gpu__time_duration.sum','dram__bytes_read.sum','dram__bytes_write.sum','sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active','sm__warps_active.avg.per_cycle_active','smsp__inst_executed.sum','smsp__issue_active.avg.per_cycle_active','launch__registers_per_thread','sm__sass_thread_inst_executed_op_dadd_pred_on.sum','sm__sass_thread_inst_executed_op_dmul_pred_on.sum','sm__sass_thread_inst_executed_op_dfma_pred_on.sum','launch__grid_size','launch__occupancy_limit_registers','sm__maximum_warps_per_active_cycle_pct']
for vals in rows[2:]:
    d=dict(zip(hdr,vals))
    print('----')
    for k in keys: print(' ',k, d.get(k,'')[:60])
    st={h.replace('smsp__pcsamp_warps_issue_stalled_',''):float(v) for h,v in d.items() if h.startswith('smsp__pcsamp_warps_issue_stalled_') and not h.endswith('not_issued') and v}
    tot=sum(st.values()) or 1; print('  stalls:', ', '.join(f"{k}={100*v/tot:.0f}%" for k,v in sorted(st.items(),key=lambda x:-x[1]) if v/tot>0.02))

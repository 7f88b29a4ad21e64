# ncu --set full of the two row kernels (one launch each) + warp-state summary
KREGEX='k_rows' NCU_COUNT=2 bash scripts/ncu_one.sh
for k in k_rows_fwd2 k_rows_bwd2; do
  echo "== $k"
  ncu -i gpurun_out/prof.ncu-rep -k regex:$k --page details --csv 2>/dev/null | python3 -c "
import csv,sys
for r in csv.reader(sys.stdin):
    if len(r)>14 and any(x in r[12] for x in ('Stall','Issue','Eligible','Active Warps','Duration','Executed Ipc','Registers','Achieved Occupancy','Theoretical Occupancy','No Eligible','Warp Cycles')): print(r[12],'|',r[14])
" | head -60
done
python3 scripts/ncu_src.py gpurun_out/prof.ncu-rep k_rows_bwd2 ttemb_fused > gpurun_out/src_bwd.txt 2>&1
python3 scripts/ncu_src.py gpurun_out/prof.ncu-rep k_rows_fwd2 ttemb_fused > gpurun_out/src_fwd.txt 2>&1
ncu -i gpurun_out/prof.ncu-rep --page raw --csv 2>/dev/null | python3 -c "
import csv,sys
rows=list(csv.reader(sys.stdin)); h=rows[0]
want=[i for i,x in enumerate(h) if x.startswith('smsp__pcsamp_warps_issue_stalled_') and not x.endswith('not_issued')]
for r in rows[2:]:
    print(r[h.index('Kernel Name')][:40])
    v=sorted(((float(r[i] or 0),h[i]) for i in want), reverse=True)[:12]
    for x,n in v: print('   ',n.replace('smsp__pcsamp_warps_issue_stalled_',''),x)
" > gpurun_out/stalls.txt 2>&1

# ncu --set full of one kernel (KREGEX) + stall / issue summary + per-line table (FSUB file)
export KREGEX=${KREGEX:-k_rows_bwd2}; NCU_COUNT=1 bash scripts/ncu_one.sh
ncu -i gpurun_out/prof.ncu-rep --page details --csv 2>/dev/null | python3 -c "
import csv,sys
for r in csv.reader(sys.stdin):
    if len(r)>14 and any(x in r[12] for x in ('Issue Slots Busy','Eligible Warps','Duration','Issued Instructions','Registers Per','Achieved Active','DRAM Throughput','Memory Throughput','L1/TEX Hit','L2 Hit')): print(r[12],'|',r[14])
"
ncu -i gpurun_out/prof.ncu-rep --page raw --csv 2>/dev/null | python3 -c "
import csv,sys
rows=list(csv.reader(sys.stdin)); h=rows[0]
want=[i for i,x in enumerate(h) if x.startswith('smsp__pcsamp_warps_issue_stalled_') and not x.endswith('not_issued')]
for r in rows[2:]:
    print(r[h.index('Kernel Name')][:40])
    v=sorted(((float(r[i] or 0),h[i]) for i in want), reverse=True)[:10]
    for x,n in v: print('   ',n.replace('smsp__pcsamp_warps_issue_stalled_',''),x)
"
python3 scripts/ncu_src.py gpurun_out/prof.ncu-rep ${KREGEX} ${FSUB:-ttemb_fused} > gpurun_out/src_k.txt 2>&1

# compute-sanitizer over small cases (memcheck / racecheck / synccheck / initcheck); summaries only
mkdir -p gpurun_out/sanitizer
for tool in memcheck racecheck synccheck initcheck; do
  for c in ${CASES:-c1 c2-b256 tc-r32 tc-r64 tc-r128 ffma-split hosttier}; do
    timeout 900 compute-sanitizer --tool $tool --print-limit 20 python scripts/sanitize_case.py $c > gpurun_out/sanitizer/${tool}_$c.log 2>&1
    echo "$tool $c rc=$? : $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' gpurun_out/sanitizer/${tool}_$c.log | tail -1)"
  done
done

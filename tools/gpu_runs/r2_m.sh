export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/sanitizer2
for w in grid1 grid2 zgetrf; do
  for t in memcheck racecheck synccheck; do
    timeout 600 compute-sanitizer --tool $t --print-limit 10 python tools/sanitize_run.py $w > gpurun_out/sanitizer2/${w}_${t}.log 2>&1
    echo "$w $t rc=$? $(grep -h 'ERROR SUMMARY\|RACECHECK SUMMARY' gpurun_out/sanitizer2/${w}_${t}.log | tr '\n' ' ') $(grep -c '^ok' gpurun_out/sanitizer2/${w}_${t}.log)"
  done
done
bash tools/gpu_runs/r2_l.sh
bash tools/gpu_runs/r2_multi.sh

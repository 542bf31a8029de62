# compute-sanitizer memcheck / racecheck / synccheck over every tier and building block (small batches)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/sanitizer
for w in tierS tierM L1 grid1 grid2 partial partial_lapack getrs getrs_vec extend_add zgetrf tree; do
  for t in memcheck racecheck synccheck; do
    timeout 600 compute-sanitizer --tool $t --print-limit 10 python tools/sanitize_run.py $w > gpurun_out/sanitizer/${w}_${t}.log 2>&1
    echo "$w $t rc=$? $(grep -h 'ERROR SUMMARY\|RACECHECK SUMMARY' gpurun_out/sanitizer/${w}_${t}.log | tr '\n' ' ') $(grep -c '^ok' gpurun_out/sanitizer/${w}_${t}.log)"
  done
done

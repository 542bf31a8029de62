# few-large: inner trailing update as a grid-wide GEMM (split_strip): tests + bench_next large
export PATH=/usr/local/cuda/bin:$PATH
O=gpurun_out/r3o; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_large.py tests/test_gpu_getrf.py -x -q -k "large_g1 or two_level or 8192" > $O/pytest.log 2>&1; echo pytest rc $?; tail -1 $O/pytest.log
timeout 900 python tools/bench_next.py --what large --reps 3 > $O/bench_large.jsonl 2> $O/bench_large.err; echo large rc $?; cut -c1-330 $O/bench_large.jsonl

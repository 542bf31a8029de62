# tier S: finer width classes (32 / 28 / 24 / 20 / ...): tests + C1big A/B (current vs previous build)
export PATH=/usr/local/cuda/bin:$PATH
O=gpurun_out/r3q; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_getrf.py -x -q -k "grouped or c1_parity or edge or g1 or singular or closed or leading" > $O/pytest.log 2>&1; echo pytest rc $?; tail -1 $O/pytest.log
for r in 1 2; do
timeout 200 python bench.py --config C1big --no-cpu-baseline --no-e2e > $O/bench_C1big_fine_r$r.json 2> $O/bench_C1big_fine_r$r.err; python -c "import json; d=json.load(open('$O/bench_C1big_fine_r$r.json')); print('C1big fine', round(d['ms_per_step'],3), round(d['roofline']['frac'],3))"
done

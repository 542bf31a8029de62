timeout 600 python -m pytest tests/test_gpu_getrf.py -x -q -k "c1_parity or edge or g1_exact or leading or singular or dominant or closed or bad_arg" > gpurun_out/pytest_s.log 2>&1; echo rc $?; tail -1 gpurun_out/pytest_s.log
for v in "4 0" "4 1" "5 1" "6 1"; do set -- $v
IRR_NVCC_EXTRA="-DIRR_S32_CTAS=$1 -DIRR_S32_SCR=$2" python -m paper_conf_sc_abdelfattahgbtld22_b200.build --force > /dev/null 2>&1
timeout 300 python bench.py --config C1big --no-cpu-baseline --no-e2e > /tmp/b.json 2>/tmp/b.err; tail -1 /tmp/b.err
python -c "import json; d=json.load(open('/tmp/b.json')); print('C1big ctas=$1 scr=$2', round(d['ms_per_step'],3), round(d['value'],1), round(d['roofline']['frac'],3))"
done

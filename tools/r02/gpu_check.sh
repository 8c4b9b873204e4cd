#!/bin/bash
# round-2 GPU session: build, smoke, full GPU suite, default bench line, R-MAT bench,
# ncu of the lean L2 probe (a steady launch)
O=gpurun_out/${TAG:-r02b}
mkdir -p $O
python -c "import __graft_entry__ as e; e.build(); e.smoke()" > $O/smoke.txt 2>&1
tail -2 $O/smoke.txt
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider ${PYTEST_ARGS} > $O/tests_gpu.txt 2>&1
tail -5 $O/tests_gpu.txt
timeout 600 python bench.py --out $O/bench_default.jsonl > $O/bench_default.log 2>&1; echo "bench rc=$?"
tail -c 400 $O/bench_default.log
for c in ${BENCH_CFGS:-rmat:64}; do
  timeout 600 python bench.py --workload ${c%%:*} --K ${c##*:} --steps 10 --no-cpu-baseline --e2e-steps 0 --out $O/bench_cfgs.jsonl > $O/bench_${c%%:*}_${c##*:}.log 2>&1; echo "bench $c rc=$?"
done
if [ "${NCU_PROBE:-1}" = "1" ]; then
timeout 300 ncu --set full --clock-control none -k regex:l2_gather_lean -s 3 -c 1 --csv --page raw python - > $O/ncu_l2_lean.csv 2>&1 <<'PY'
import ctypes, __graft_entry__
lp = ctypes.CDLL(__graft_entry__.build_l2_probe())
g, m = ctypes.c_float(), ctypes.c_float()
lp.l2_probe_read_gbs2(ctypes.c_int64(48 << 20), ctypes.c_int32(256), ctypes.c_int32(2), ctypes.byref(g), ctypes.byref(m))
PY
fi

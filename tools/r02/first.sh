#!/bin/bash
# round-2 first GPU session: baseline bench, L2 probe variants, R-MAT knob sweep
mkdir -p gpurun_out/r02a
O=gpurun_out/r02a
python -c "import __graft_entry__ as e; e.build()" > $O/build.txt 2>&1
timeout 600 python bench.py --out $O/bench_default.jsonl > $O/bench_default.log 2>&1
python - > $O/l2probe.txt 2>&1 <<'PY'
import ctypes, __graft_entry__
lp = ctypes.CDLL(__graft_entry__.build_l2_probe())
for mb in (32, 48, 64, 96):
    for mode in (0, 1, 2, 3):
        for rb in ((256, 512) if mode in (0, 2) else (256,)):
            g, m = ctypes.c_float(), ctypes.c_float()
            rc = lp.l2_probe_read_gbs2(ctypes.c_int64(mb << 20), ctypes.c_int32(rb), ctypes.c_int32(mode), ctypes.byref(g), ctypes.byref(m))
            print("MB=%d mode=%d row=%d rc=%d GB/s=%.0f ms=%.3f" % (mb, mode, rb, rc, g.value, m.value), flush=True)
PY
for ipp in 0 256 512 1024; do
  timeout 300 python bench.py --workload rmat --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-cusparse --no-l2-probe --items-per-part $ipp --out $O/rmat_ipp.jsonl > /dev/null 2>&1
done
for e in "MPS_MAX_W=2" "MPS_DYN=0" "MPS_MAX_W=2 MPS_DYN=0"; do
  env $e timeout 300 python bench.py --workload rmat --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-cusparse --no-l2-probe --out $O/rmat_env_${e// /_}.jsonl > /dev/null 2>&1
done
for wl in cora:16 pubmed:64; do
  timeout 300 python bench.py --workload ${wl%%:*} --K ${wl##*:} --cuda-graph --steps 20 --warmup 5 --e2e-steps 0 --no-cpu-baseline --no-l2-probe --out $O/tiny_graph.jsonl > /dev/null 2>&1
done
timeout 300 ncu --set full --clock-control none -k regex:l2_gather_lean -c 1 --csv --page raw python - > $O/ncu_l2_lean.csv 2>&1 <<'PY'
import ctypes, __graft_entry__
lp = ctypes.CDLL(__graft_entry__.build_l2_probe())
g, m = ctypes.c_float(), ctypes.c_float()
lp.l2_probe_read_gbs2(ctypes.c_int64(48 << 20), ctypes.c_int32(256), ctypes.c_int32(2), ctypes.byref(g), ctypes.byref(m))
PY
ls -la $O

#!/bin/bash
O=gpurun_out/r02g; mkdir -p $O
python - > $O/tma_gather.txt 2>&1 <<'PY'
import ctypes
lp = ctypes.CDLL("tools/libtmagather.so")
l2 = ctypes.CDLL("tools/libl2probe.so")
for mb in (32, 48, 64, 96, 256, 1024):
    g, m, c = ctypes.c_float(), ctypes.c_float(), ctypes.c_int()
    rc = lp.tma_gather_probe_gbs(ctypes.c_int64(mb << 20), ctypes.byref(g), ctypes.byref(m), ctypes.byref(c))
    g2, m2 = ctypes.c_float(), ctypes.c_float()
    rc2 = l2.l2_probe_read_gbs2(ctypes.c_int64(mb << 20), ctypes.c_int32(256), ctypes.c_int32(2), ctypes.byref(g2), ctypes.byref(m2))
    print("MB=%d tma_gather4 rc=%d GB/s=%.0f cfg=%d | lsu lean gather rc=%d GB/s=%.0f" % (mb, rc, g.value, c.value, rc2, g2.value), flush=True)
PY
cat $O/tma_gather.txt
timeout 300 ncu --set full --clock-control none -k regex:tma_gather_kernel -s 2 -c 1 --csv --page raw python - > $O/ncu_tma_gather.csv 2>&1 <<'PY'
import ctypes
lp = ctypes.CDLL("tools/libtmagather.so")
g, m, c = ctypes.c_float(), ctypes.c_float(), ctypes.c_int()
lp.tma_gather_probe_gbs(ctypes.c_int64(48 << 20), ctypes.byref(g), ctypes.byref(m), ctypes.byref(c))
PY
python tools/ncu_summary.py $O/ncu_tma_gather.csv 2>&1 | head -25

#!/bin/bash
O=gpurun_out/r02i; mkdir -p $O
python -c "import __graft_entry__ as e; e.build()" > $O/build.txt 2>&1
python - > $O/async_probe.txt 2>&1 <<'PY'
import ctypes
l2 = ctypes.CDLL("tools/libl2probe.so")
for mb in (32, 48, 96, 256, 1024):
    out = []
    for mode in (2, 4):
        g, m = ctypes.c_float(), ctypes.c_float()
        rc = l2.l2_probe_read_gbs2(ctypes.c_int64(mb << 20), ctypes.c_int32(256), ctypes.c_int32(mode), ctypes.byref(g), ctypes.byref(m))
        out.append("mode%d rc=%d %.0f" % (mode, rc, g.value))
    print("MB=%d" % mb, " | ".join(out), flush=True)
PY
cat $O/async_probe.txt

#!/bin/bash
# r02ap: NVRTC repeat-compile speedup on the box: in-process only, or persistent across processes?
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
(
echo "== before: ~/.nv"; du -sh ~/.nv 2>/dev/null; ls -la ~/.nv/ComputeCache 2>/dev/null | head -5
echo "== process 1"; timeout 300 python scripts/nvrtc_repeat_probe.py
echo "== after p1: ~/.nv"; du -sh ~/.nv 2>/dev/null; find ~/.nv -newer scripts/nvrtc_repeat_probe.py -type f 2>/dev/null | head -5
echo "== process 2"; timeout 300 python scripts/nvrtc_repeat_probe.py
echo "== process 3, HOME elsewhere"; HOME=$(mktemp -d) timeout 300 python scripts/nvrtc_repeat_probe.py
echo "== strace-free check: files opened"; ls -la /tmp | head -20
python -c "import ctypes,glob; l=ctypes.CDLL(sorted(glob.glob('/usr/local/cuda/lib64/libnvrtc.so*'))[0]); a=ctypes.c_int(); b=ctypes.c_int(); l.nvrtcVersion(ctypes.byref(a),ctypes.byref(b)); print('nvrtc', a.value, b.value)"
nproc; cat /proc/cpuinfo | grep "model name" | head -1
) 2>&1 | tee gpurun_out/nvrtc_cache_probe_r02ap.txt

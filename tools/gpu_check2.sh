#!/bin/bash
# cuFile probe (opt-in path), FILE tests, HotSpot v4 tests + throughput, default bench line with staging/e2e roofline.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 90 python tools/cufile_probe.py > gpurun_out/cufile_probe.log 2>&1; echo "cufile probe rc=$?"; tail -8 gpurun_out/cufile_probe.log
ls /etc/cufile.json 2>&1; ls /dev/nvidia-fs* 2>&1 | head -2; lsmod 2>/dev/null | grep -i nvidia_fs
timeout 600 python -m pytest tests/test_gpu_file.py -q -x > gpurun_out/tg_file.log 2>&1; tail -2 gpurun_out/tg_file.log | cut -c1-300
bash tools/gpu_hs_v4.sh
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; echo "bench rc=$?"

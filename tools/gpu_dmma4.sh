mkdir -p gpurun_out
timeout 600 python tools/f64_probe.py 8192 > gpurun_out/g_f64.txt 2>&1
timeout 1500 python -m pytest tests/test_gpu_f64.py tests/test_gpu_apps.py tests/test_gpu_faults.py tests/test_gpu_shard.py tests/test_gpu_fullsize.py -m gpu -q -x -p no:cacheprovider > gpurun_out/g_tests.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_dmma_kernel -c 1 -o gpurun_out/g_dmma python tools/f64_probe.py 8192 > gpurun_out/g_ncu.log 2>&1
echo done

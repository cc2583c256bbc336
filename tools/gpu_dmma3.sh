mkdir -p gpurun_out
timeout 600 python tools/f64_probe.py 8192 > gpurun_out/f_f64_w16.txt 2>&1
PS_DMMA_WARPS=8 timeout 600 python tools/f64_probe.py 8192 > gpurun_out/f_f64_w8.txt 2>&1
timeout 1500 python -m pytest tests/test_gpu_f64.py tests/test_gpu_apps.py tests/test_gpu_faults.py tests/test_gpu_shard.py -m gpu -q -x -p no:cacheprovider > gpurun_out/f_tests.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/f_bench.json 2> gpurun_out/f_bench.err
echo done

mkdir -p gpurun_out
timeout 600 python tools/f64_probe.py 8192 > gpurun_out/h_f64_v0.txt 2>&1
PS_DMMA_VARIANT=1 timeout 600 python tools/f64_probe.py 8192 > gpurun_out/h_f64_v1.txt 2>&1
timeout 1500 python -m pytest tests/test_gpu_f64.py tests/test_gpu_apps.py tests/test_gpu_faults.py -m gpu -q -x -p no:cacheprovider > gpurun_out/h_tests.log 2>&1
echo done

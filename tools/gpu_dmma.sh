mkdir -p gpurun_out
timeout 300 ./tools/dmma_probe > gpurun_out/d_probe.txt 2>&1
timeout 600 python tools/f64_probe.py 8192 > gpurun_out/d_f64_dmma.txt 2>&1
PS_F64_DFMA=1 timeout 600 python tools/f64_probe.py 8192 > gpurun_out/d_f64_dfma.txt 2>&1
timeout 1200 python -m pytest tests/test_gpu_apps.py tests/test_gpu_faults.py tests/test_gpu_fullsize.py tests/test_gpu_shard.py -m gpu -q -x -p no:cacheprovider > gpurun_out/d_tests.log 2>&1
echo done

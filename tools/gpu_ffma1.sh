mkdir -p gpurun_out
timeout 600 python tools/f32_probe.py 8192 > gpurun_out/k_f32_new.txt 2>&1
PS_F32_SIMT_OLD=1 timeout 600 python tools/f32_probe.py 8192 > gpurun_out/k_f32_old.txt 2>&1
timeout 600 python tools/f64_probe.py 8192 > gpurun_out/k_f64.txt 2>&1
timeout 1500 python -m pytest tests/test_gpu_f64.py tests/test_gpu_apps.py tests/test_gpu_faults.py tests/test_gpu_shard.py tests/test_gpu_fullsize.py tests/test_gpu_sanitizer.py -m gpu -q -x -p no:cacheprovider > gpurun_out/k_tests.log 2>&1
echo done

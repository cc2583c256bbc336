mkdir -p gpurun_out
for v in 3 4 0; do PS_DMMA_VARIANT=$v timeout 600 python tools/f64_probe.py 8192 > gpurun_out/i_f64_v$v.txt 2>&1; done
echo done

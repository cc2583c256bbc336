#!/bin/bash
# tcgen05 B-majorness experiment: N-major B (default) vs K-major B (PS_TC_BT=1:
# a transposed copy, its time included in kernel_ms), GEMM 8192^3 per dtype.
python tools/tc8_probe.py 8192 5
PS_TC_BT=1 python tools/tc8_probe.py 8192 5

echo "== normal"; timeout 60 python tools/conv_trace.py 6e_1x1 7c_1x1 | grep -E "==|mma_end|cta0 full"
echo "== no MMA"; HIOS_DBG=1 timeout 60 python tools/conv_trace.py 6e_1x1 7c_1x1 | grep -E "==|mma_end|cta0 full"
echo "== no TMA"; HIOS_DBG=2 timeout 60 python tools/conv_trace.py 6e_1x1 7c_1x1 | grep -E "==|mma_end|cta0 full"
echo "== neither"; HIOS_DBG=3 timeout 60 python tools/conv_trace.py 6e_1x1 7c_1x1 | grep -E "==|mma_end|cta0 full"

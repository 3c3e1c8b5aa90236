nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout 400 python -m pytest tests -m gpu -q -rf -k "digitize or fp32" -p no:cacheprovider > gpurun_out/t_fp32.log 2>&1
echo "exit $?" >> gpurun_out/t_fp32.log
timeout 400 python -m pytest tests -m gpu -q -rf -x -k "tc_f16_tolerance and 255" -p no:cacheprovider > gpurun_out/t_tc1.log 2>&1
echo "exit $?" >> gpurun_out/t_tc1.log
timeout 600 python -m pytest tests -m gpu -q -rf -k "not digitize and not fp32" -p no:cacheprovider > gpurun_out/t_rest.log 2>&1
echo "exit $?" >> gpurun_out/t_rest.log

timeout 300 python tools/time_list.py > gpurun_out/time_list.log 2>&1
for v in spt2 spt4 cs1 spt2cs1; do B2CL_LIB=build/variants/$v.so timeout 300 python tools/time_list.py >> gpurun_out/time_list.log 2>&1; done
timeout 600 python -m pytest tests/test_gpu_sampling.py tests/test_gpu_arrays.py -m gpu -x -q > gpurun_out/t_list.log 2>&1; echo rc=$? >> gpurun_out/t_list.log
B2CL_LIB=build/variants/spt4.so timeout 600 python -m pytest tests/test_gpu_sampling.py tests/test_gpu_arrays.py -m gpu -x -q > gpurun_out/t_list4.log 2>&1; echo rc=$? >> gpurun_out/t_list4.log

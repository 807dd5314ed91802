cd $GRAFT_REPO_ROOT
nvidia-smi --query-gpu=name,memory.total,clocks.max.sm,pcie.link.gen.max,pcie.link.width.max --format=csv > gpurun_out/gpu_info.txt 2>&1
python -c "import torch; p=torch.cuda.get_device_properties(0); print(p, p.multi_processor_count)" >> gpurun_out/gpu_info.txt 2>&1
lscpu | head -20 >> gpurun_out/gpu_info.txt
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke exit $?" >> gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
tail -5 gpurun_out/smoke.log; tail -30 gpurun_out/pytest_gpu.log

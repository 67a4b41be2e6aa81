mkdir -p gpurun_out
python __graft_entry__.py
(python tools/dag_timing.py C2; FELIX_DPHI_BN=96 python tools/dag_timing.py C2; FELIX_CHAIN_CS=1 python tools/dag_timing.py C2; python tools/dag_timing.py C2 8192; FELIX_DPHI_BN=96 python tools/dag_timing.py C2 8192) > gpurun_out/dphi5.log 2>&1
(timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "eval_parity or one_adam or modes or full_size or multitask" 2>&1 | tail -5) > gpurun_out/t5.log

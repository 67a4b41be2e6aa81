mkdir -p gpurun_out
python __graft_entry__.py
(timeout 900 python -m pytest tests/test_gpu_parity.py -q -s -k "split_cone" 2>&1 | tail -6) > gpurun_out/t21.log
for cfg in "4 4 1" "8 4 1" "8 4 2" "8 2 2" "4 2 2" "8 2 4" "4 4 2" "8 1 4"; do set -- $cfg; (echo "P=$1 W=$2 G=$3"; FELIX_P=$1 FELIX_SCW=$2 FELIX_SCG=$3 timeout 120 python tools/dag_timing.py C2) >> gpurun_out/dag21.log 2>&1; done
for cfg in "2 8 1" "2 8 2" "4 8 1" "4 4 2"; do set -- $cfg; (echo "C5 P=$1 W=$2 G=$3"; FELIX_P=$1 FELIX_SCW=$2 FELIX_SCG=$3 timeout 120 python tools/dag_timing.py C5) >> gpurun_out/dag21.log 2>&1; done

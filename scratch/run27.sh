mkdir -p gpurun_out
python __graft_entry__.py
for cfg in "4 2" "4 1" "2 2" "2 1" "8 2"; do set -- $cfg; (echo "C2 P=$1 R=$2"; FELIX_P=$1 FELIX_R=$2 timeout 120 python tools/dag_timing.py C2) >> gpurun_out/dag27.log 2>&1; done
for cfg in "2 2" "4 2" "1 2"; do set -- $cfg; (echo "C2@16384 P=$1 R=$2"; FELIX_P=$1 FELIX_R=$2 timeout 120 python tools/dag_timing.py C2 16384) >> gpurun_out/dag27.log 2>&1; done

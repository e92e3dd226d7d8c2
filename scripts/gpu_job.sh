set -x
bash scripts/gpu_quick.sh
TOPK=k_lane_problems bash scripts/gpu_ncu_top.sh

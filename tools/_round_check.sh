# one gpurun call: build + GPU tests + smoke + bench + reference arm (gpu_check.sh), then the
# round's profile artifacts (profile_round.sh); results under gpurun_out/$1 and gpurun_out/$1_prof
bash tools/gpu_check.sh ${1:-check}
bash tools/profile_round.sh ${1:-check}_prof

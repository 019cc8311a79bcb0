#!/bin/bash
# One gpurun session: bench line, ncu launch list of the same command, ncu --set full of each kernel.
# usage (on the box): bash tools/gpu_profile_round.sh <tag> [kernels...]
TAG=${1:-r01}; shift
KERNELS=${@:-"nbody1m nbody1m_p8 nbody4096 sim4096 nbody64 bs_map bs_fused mandel matmul reduce cp mriq series idea"}
mkdir -p gpurun_out
python bench.py > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err
echo "bench rc=$?"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}.csv \
    python bench.py --steps 3 --warmup 3 > gpurun_out/bench_under_ncu_${TAG}.json 2>&1
echo "launch list rc=$?"
declare -A KRE=( [nbody1m]=force_kernel [nbody1m_p8]=force_kernel [nbody4096]=force_ [nbody64]=force64_kernel [series]=series_kernel [sim4096]=simulate_small [idea]=idea_kernel [bs_map]=map_kernel
                 [bs_fused]=map_reduce_kernel [mandel]=mandel_kernel [matmul]=gemm [reduce]=reduce_kernel [cp]=bmap_kernel [mriq]=bmap_kernel )
# skip counts: the 2^20 force map is two force_kernel launches per call (mass-uniform splits, then
# the rest; R11) -- skip 2 captures the second call's mass-uniform launch
declare -A SKIP=( [nbody1m]=2 [nbody1m_p8]=2 )
for k in $KERNELS; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:${KRE[$k]} -s ${SKIP[$k]:-1} -c 1 \
      -o gpurun_out/prof_${k}_${TAG} -f python tools/prof_kernels.py $k 2 > gpurun_out/prof_${k}_${TAG}.log 2>&1
  echo "prof $k rc=$?"
done
# summaries on the box (the .ncu-rep files of a full round exceed what gpurun brings back)
mkdir -p gpurun_out/prof_${TAG}; PROF_DIR=gpurun_out/prof_${TAG} python tools/make_profiles.py ${TAG} > gpurun_out/prof_${TAG}/make_profiles.log 2>&1
cp gpurun_out/launches_${TAG}.csv gpurun_out/bench_${TAG}.json gpurun_out/prof_${TAG}/ 2>/dev/null
if [ -z "$KEEP_REPS" ]; then rm -f gpurun_out/prof_*_${TAG}.ncu-rep; fi

#!/bin/bash
# Round-2 session u: why the warp-specialised kernel is fast for Adam N = 8 and slow for N = 6 / 7 -- one ncu --set full
# capture each (U = 2), their warp-state and occupancy sections.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for n in 6 7 8; do
  timeout 900 ncu --set full --clock-control none -k regex:colocated -s 3 -c 1 -o gpurun_out/ws_adam$n -f \
      python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --optimizer adam --n $n --variant warpspec > gpurun_out/ws_adam$n.log 2>&1
  ncu -i gpurun_out/ws_adam$n.ncu-rep --page details --section WarpStateStats --section Occupancy --section LaunchStats \
      --section SpeedOfLight --section MemoryWorkloadAnalysis > gpurun_out/ws_adam${n}_details.txt 2>&1
  ncu -i gpurun_out/ws_adam$n.ncu-rep --page raw --csv > gpurun_out/ws_adam${n}_raw.csv 2>/dev/null
done
rm -f gpurun_out/*.ncu-rep
grep -E "Stall|Warp Cycles|Achieved Occupancy|Block Limit|Duration|DRAM Throughput|Registers|Waves" gpurun_out/ws_adam*_details.txt | head -80
echo session done

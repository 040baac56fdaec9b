#!/bin/bash
# Round-end evidence at HEAD (under gpurun): sanitizers on smoke(), ncu --set full of the POTRF tile
# launches, the ncu launch list of one timed factorisation (n = 32768).
mkdir -p gpurun_out
timeout 600 compute-sanitizer --tool memcheck --leak-check no python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/sanitize_memcheck.txt 2>&1; echo "memcheck rc=$?"; tail -1 gpurun_out/sanitize_memcheck.txt
timeout 600 compute-sanitizer --tool synccheck python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/sanitize_synccheck.txt 2>&1; echo "synccheck rc=$?"; tail -1 gpurun_out/sanitize_synccheck.txt
timeout 900 compute-sanitizer --tool racecheck python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/sanitize_racecheck.txt 2>&1; echo "racecheck rc=$?"; tail -1 gpurun_out/sanitize_racecheck.txt
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"dataflow|bulk" -s 2 -c 2 -f \
    -o gpurun_out/prof_potrf_tile python tools/prof_kernel.py 3 1024 1024 0 1 > gpurun_out/prof_potrf_tile.log 2>&1; echo "prof potrf rc=$?"
python tools/ncu_summary.py gpurun_out/prof_potrf_tile.ncu-rep potrf_tile > gpurun_out/ncu_summary_potrf.txt 2>&1
timeout 1500 bash tools/launchlist.sh --order 32768 --tile 1024 > gpurun_out/launchlist.log 2>&1; echo "launchlist rc=$?"
tail -25 gpurun_out/launches_summary.txt

bash tools/prof_round.sh > gpurun_out/prof_round.log 2>&1
timeout 1500 bash tools/launchlist.sh > gpurun_out/launchlist.log 2>&1
gzip -f gpurun_out/launches.csv

make -j16 > gpurun_out/make.log 2>&1
timeout 1200 python experiments.py sweep > gpurun_out/sweep.log 2>&1; echo "sweep rc=$?"; tail -c 1500 gpurun_out/sweep.log
timeout 1800 python experiments.py kbe > gpurun_out/kbe.log 2>&1; echo "kbe rc=$?"; tail -c 1500 gpurun_out/kbe.log

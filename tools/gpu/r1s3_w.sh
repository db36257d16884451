make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
P="python tools/pin_shape.py Q7 100 4096 3 8 1 1 8192"
timeout -s KILL 300 $P
GPL_OPTS=lazy_columns=0 timeout -s KILL 300 python tools/pin_shape.py Q7 100 2048 3 8 1 1 8192
GPL_OPTS=clustered=0 timeout -s KILL 300 $P
GPL_OPTS=lazy_columns=1 timeout -s KILL 300 $P
timeout -s KILL 300 python tools/pin_shape.py Q7 100 4096 3 8 1 2 8192
timeout -s KILL 300 python tools/pin_shape.py Q7 100 2048 3 12 1 1 8192
timeout -s KILL 300 python tools/pin_shape.py Q7 100 1024 4 15 2 1 4096

#!/bin/bash
TAG=${TAG:-m8} bash tools/gpu_knobs.sh
TAG=${TAG:-m8} QS="Q5 Q7 Q8 Q9 Q14" bash tools/gpu_m6.sh

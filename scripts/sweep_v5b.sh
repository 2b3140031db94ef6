#!/bin/bash
V="--variant 5 --tile-rows 4"
bash scripts/sweep.sh v5sweep2 "-|$V --stages 4" "-|$V --stages 6" "t_m2u3|$V --stages 6" "t_m2u3|$V --stages 8" "t_m2u2|$V --stages 6" "t_m3u3|$V --stages 4" "t_m3u3|$V --stages 6" "t_m2u3np|$V --stages 6" "t_m2u3|--variant 5 --tile-rows 3 --stages 6" "t_m2u3|--variant 5 --tile-rows 2 --stages 6" "-|--variant 5 --tile-rows 2 --stages 4" "-|--variant 5 --tile-rows 3 --stages 4"

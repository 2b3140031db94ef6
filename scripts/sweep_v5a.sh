#!/bin/bash
V="--variant 5 --tile-rows 4"
bash scripts/sweep.sh v5sweep "-|$V" "-|$V --stages 4" "-|$V --stages 6" "t_m3u1|$V --stages 4" "t_m2u2|$V --stages 4" "t_m2u2|$V --stages 6" "t_m2u2|$V --stages 8" "t_m2u1|$V --stages 4" "t_m2u1|$V --stages 6" "t_m2u1|$V --stages 8" "t_m2u1|$V --stages 4 --block-x 128" "t_m2u1|$V --stages 6 --block-x 128" "t_m2u2|$V --stages 6 --block-x 128" "-|$V --stages 4 --block-x 128" "t_m2u1|--variant 5 --tile-rows 3 --stages 6" "-|--variant 5 --tile-rows 3 --stages 4"

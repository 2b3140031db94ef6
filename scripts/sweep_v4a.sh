#!/bin/bash
bash scripts/sweep.sh v4sweep "-|--variant 1" "-|--variant 4" "u3m4|--variant 4" "u1m3|--variant 4" "u1m3|--variant 4 --stages 4" "u2m3|--variant 4" "u2m3|--variant 4 --stages 4" "u3m3|--variant 4" "u3m3|--variant 4 --stages 4" "u3m3|--variant 4 --stages 5" "-|--variant 4 --stages 4" "-|--variant 4 --stages 2"

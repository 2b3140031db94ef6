#!/bin/bash
bash scripts/sweep.sh v5sweep5 "-|" "-|--block-x 128 --stages 6" "-|--block-x 128 --stages 8" "-|--block-x 192 --stages 6" "-|--block-x 192 --stages 8" "-|--block-x 224 --stages 8" "-|--block-x 160 --stages 8" "-|--stages 7" "-|--stages 9"

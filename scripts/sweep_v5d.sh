#!/bin/bash
bash scripts/sweep.sh v5sweep4 "shrink128|" "shrink160|" "shrink200|" "shrink256|" "shrink320|" "shrink200|--blocks-per-sm 1 --stages 16"

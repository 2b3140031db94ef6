#!/bin/bash
bash scripts/sweep.sh v5sweep3 "-|" "shrink32|" "shrink64|" "shrink96|" "shrink128|" "-|--stages 10" "-|--stages 12" "shrink64|--stages 10"

VARIANTS="1 1024 1,1 512 1,1 256 1" bash scripts/ab_lastframe.sh

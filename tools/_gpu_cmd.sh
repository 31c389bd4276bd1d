export PYTHONUNBUFFERED=1
C2="tile_x=64,threads=128,block_x=1,block_y=1,block_cby=4,tile_y=8,zchunk=32
tile_x=64,threads=128,block_x=1,block_y=4,block_cby=1,tile_y=8,zchunk=32
tile_x=64,threads=128,block_x=2,block_y=2,block_cby=1,tile_y=8,zchunk=32
tile_x=64,threads=64,block_x=2,block_y=2,block_cby=2,tile_y=8,zchunk=32
tile_x=64,threads=128,block_x=2,block_y=2,block_cby=2,tile_y=16,zchunk=32
tile_x=32,threads=64,block_x=2,block_y=4,block_cby=1,tile_y=16,zchunk=32
tile_x=64,threads=128,block_x=1,block_y=2,block_cby=2,tile_y=8,zchunk=32"
args=""; for c in $C2; do args="$args --cfg $c --cfg $c,zqueue=0"; done
timeout 500 python tools/sweep.py C2 --group 0 $args > gpurun_out/sw12_c2.log 2>&1
C4="tile_x=32,threads=256,block_x=1,block_y=1,block_cby=2,tile_y=16,zchunk=16
tile_x=32,threads=128,block_x=1,block_y=1,block_cby=4,tile_y=16,zchunk=16
tile_x=32,threads=128,block_x=2,block_y=2,block_cby=1,tile_y=16,zchunk=16
tile_x=64,threads=128,block_x=2,block_y=2,block_cby=1,tile_y=8,zchunk=16
tile_x=32,threads=64,block_x=2,block_y=2,block_cby=2,tile_y=16,zchunk=16"
args=""; for c in $C4; do args="$args --cfg $c --cfg $c,zqueue=0"; done
timeout 900 python tools/sweep.py C4 --group 0 --plan configs/c4_plan_v3big.json $args > gpurun_out/sw12_c4g0.log 2>&1
timeout 600 python tools/sweep.py C4 --group 6 --plan configs/c4_plan_v3big.json $args > gpurun_out/sw12_c4g6.log 2>&1
tail -3 gpurun_out/sw12_c2.log

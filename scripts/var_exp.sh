# rebuild with each -D define (make -B: the flags are not a make dependency)
# and time the K = 8 wavefront schedules; the default build is restored at the end.
#   bash scripts/var_exp.sh JW_TILE_ROWS=32 JW_TAIL=5 ...
mkdir -p gpurun_out/var
for d in "$@"; do
  tag=$(echo $d | tr -c 'A-Za-z0-9' '_')
  make -B CC_DEFS="-D$d" > gpurun_out/var/build_$tag.log 2>&1 || { tail -5 gpurun_out/var/build_$tag.log; continue; }
  timeout 600 python scripts/exp_jwave.py gpurun_out/var/exp_$tag.json 8 > gpurun_out/var/exp_$tag.log 2>&1
  echo "== $d"; head -1 gpurun_out/var/exp_$tag.log; grep -E "agent-col'|default'|identity'" gpurun_out/var/exp_$tag.log | cut -c1-60
done
make -B > /dev/null 2>&1

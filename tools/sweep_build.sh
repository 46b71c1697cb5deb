#!/bin/bash
# build tuning variants into variants/<name>/libefg.so (shipped to the GPU box by gpurun)
# usage: tools/sweep_build.sh "name:-DA=1 -DB=2" ...
ROOT=$(cd "$(dirname "$0")/.." && pwd)
for spec in "$@"; do
  NAME=${spec%%:*}; DEFS=${spec#*:}
  ( bash $ROOT/tools/build_variant.sh $NAME "$DEFS" > /tmp/var_$NAME.log 2>&1 && mkdir -p $ROOT/variants/$NAME && cp $ROOT/build/var_$NAME/libefg.so $ROOT/variants/$NAME/ && echo "built $NAME" || { echo "FAILED $NAME"; grep -m3 error /tmp/var_$NAME.log; } ) &
done
wait

# build libglb.so of git revision $1 (or the working tree: WT) into build/ab/libglb_$1$TAG.so
# for GLB_LIBRARY A/B runs; extra nvcc flags in $ABFLAGS (e.g. -DGLB_KHOP_ROUNDS=2), name
# suffix in $TAG
set -e
REV=$1
D=$(mktemp -d)
if [ "$REV" = WT ]; then
  mkdir -p $D/paper_conf_eurosys_yangtswycyz22_b200
  cp -r paper_conf_eurosys_yangtswycyz22_b200/csrc $D/paper_conf_eurosys_yangtswycyz22_b200/
  cp -r include $D/
else
  git archive $REV paper_conf_eurosys_yangtswycyz22_b200/csrc include | tar -x -C $D
fi
mkdir -p build/ab
for f in $D/paper_conf_eurosys_yangtswycyz22_b200/csrc/*.cu; do
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -I$D/include --expt-relaxed-constexpr $ABFLAGS -c $f -o $D/$(basename $f .cu).o &
done
wait
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o build/ab/libglb_$REV$TAG.so $D/*.o -lcudart
rm -rf $D
echo build/ab/libglb_$REV$TAG.so

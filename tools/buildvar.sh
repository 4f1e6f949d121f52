# usage: tools/buildvar.sh <git-rev|WORK> <name>: build libtfhe_b200.so of that source state into scratch/lib_<name>.so
set -e
D=/tmp/bv_$2; rm -rf $D; mkdir -p $D/pkg
if [ "$1" = WORK ]; then cp -r /root/repo/paper_conf_ispass_maxw23_b200/csrc $D/pkg/; cp -r /root/repo/include $D/; else
  (git archive $1 paper_conf_ispass_maxw23_b200/csrc include | tar -x -C $D && mv $D/paper_conf_ispass_maxw23_b200/csrc $D/pkg/csrc); fi
nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -shared -cudart static $3 -o /root/repo/scratch/lib_$2.so $D/pkg/csrc/tb_lib.cu

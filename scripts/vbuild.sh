# usage: vbuild.sh name unit.cu [DEFS...]  -> libsand_name.so with only `unit` recompiled
name=$1; unit=$2; shift 2
P=/root/repo/paper_conf_sosp_yelllhkh25_b200; B=$P/build_$name; mkdir -p $B
defs=""; for d in "$@"; do defs="$defs -D$d"; done
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xptxas -v --expt-relaxed-constexpr $defs -I /root/repo/include -I $P/csrc -c $P/csrc/$unit -o $B/$unit.o 2> $B/ptxas.log || { tail $B/ptxas.log; exit 1; }
objs=""; for o in $P/build/*.o; do b=$(basename $o); if [ "$b" = "$unit.o" ]; then objs="$objs $B/$unit.o"; else objs="$objs $o"; fi; done
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -shared -Xcompiler -fPIC $objs -o $P/libsand_$name.so -lcudart -lpthread
grep -A1 "k_plainILi1ELi1ELi2ELb1E" $B/ptxas.log | grep -o "Used [0-9]* registers.*" | head -2

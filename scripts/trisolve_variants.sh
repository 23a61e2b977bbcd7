set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
cp paper_conf_icpp_0002s22_b200/liblf.so /tmp/lf_32_8.so
for v in "16 16" "16 8" "32 16"; do set -- $v
  LF_EXTRA_FLAGS="-DLF_TS_PK=$1 -DLF_TS_CB=$2" python -c "from paper_conf_icpp_0002s22_b200 import _build; _build.build(force=True)" > /dev/null 2>&1
  cp paper_conf_icpp_0002s22_b200/liblf.so /tmp/lf_$1_$2.so
done
for f in /tmp/lf_32_8.so /tmp/lf_16_16.so /tmp/lf_16_8.so /tmp/lf_32_16.so; do
  LF_LIB_PATH=$f python scripts/trisolve_probe.py --time
done
LF_LIB_PATH=/tmp/lf_16_16.so timeout 300 python -m pytest tests/test_gpu_trisolve.py -q 2>&1 | tail -2

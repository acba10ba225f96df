# Diagnostic: per-op times of IMC under the diagnostic builds.
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
for v in libdjinn libdjinn_nomma; do DJINN_LIB=$L/$v.so timeout 120 python tools/op_times.py imc bf16 1024 10 | grep -E "conv|fc|total"; done
DJINN_LIB=$L/libdjinn_stats.so timeout 300 python tools/run_app.py imc bf16 1024 1 2>&1 | grep "\[tc" | head -6

# Diagnostic: per-op times of IMC / FACE (tools/op_times.py); DJINN_LIB selects a variant build.
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
timeout 120 python tools/op_times.py imc bf16 1024 10 | grep -E "pool|total"
timeout 120 python tools/op_times.py face bf16 256 10 | grep -E "pool|M2|total"

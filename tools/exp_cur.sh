bash tools/ab.sh "base:libspinfer_base.so:" "scanspin:libspinfer_scanspin.so:" "consspin:libspinfer_consspin.so:"

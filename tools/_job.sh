bash tools/gpu.sh h30 build smoke suite

#include "astitch_device.cuh"
